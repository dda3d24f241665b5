"""dist.scan_sharded / dist.delta_encode_sharded END TO END with two processes (world size 2,
gloo group, payloads staged through host memory) sharing one GPU: every multi-GPU code path of
the product -- shard offsets, sam_shard_state, the payload all-gather, the device fold and the
seeded sam_shard_scan, issued on a non-default stream -- against the oracle.
On a multi-GPU box the same functions run over NCCL; only the transport differs."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _worker(rank, world, port, name, k, s, lens, q):
    try:
        import sys

        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import oracle
        import synth
        from paper_conf_pldi_malekiyb16_b200.dist import delta_encode_sharded, scan_sharded

        n = sum(lens)
        x = synth.make(n, name, "uniform", seed=99 + k + s)
        g0 = sum(lens[:rank])
        xl = torch.from_numpy(x[g0:g0 + lens[rank]].copy()).cuda()
        st = torch.cuda.Stream()
        ok = True
        for incl in (True, False):
            y = scan_sharded(xl, k, s, incl, stream=st)  # offsets from an all-gather of the lengths
            st.synchronize()
            ref = oracle.scan(x, k, s, incl)[0][g0:g0 + lens[rank]]
            ok &= bool(np.array_equal(y.cpu().numpy().view(ref.dtype), ref))
        d = delta_encode_sharded(xl, k, s, stream=st)
        st.synchronize()
        dref = oracle.delta(x, k, s)[g0:g0 + lens[rank]]
        ok &= bool(np.array_equal(d.cpu().numpy().view(dref.dtype), dref))
        q.put((rank, ok, None))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback

        q.put((rank, False, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("name,k,s,lens", [("i64", 4, 4, [1_000_003, 2_333_333]), ("i32", 2, 3, [7, 500_001]),
                                           ("i32", 8, 1, [300_001, 1]), ("i64", 1, 5, [123_457, 654_321])])
def test_two_rank_scan_sharded_end_to_end(name, k, s, lens):
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, k, s, lens, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, ok, err in sorted(res):
        assert ok, f"rank {rank}: {err}"
