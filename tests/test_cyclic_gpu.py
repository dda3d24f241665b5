"""Block-cyclic multi-GPU scan on the GPU against the oracle.

scan_cyclic_virtual runs p virtual ranks in one process on one GPU through the SAME per-rank
schedule as dist.scan_cyclic (state pass per chunk, round exchange, sam_cyclic_fold, seeded scan);
the exchange is a concatenation made once every rank has sent the round, so no kernel waits on
another rank's kernel.  The two-process test runs dist.scan_cyclic end to end over a gloo group
(payloads staged through host memory) on one GPU; on a multi-GPU box the same function runs over
NCCL."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
from tests.helpers import compare  # noqa: E402

pytestmark = pytest.mark.gpu


def _run(name, k, s, n, chunk, p, incl, lookahead=1, kind="uniform"):
    from paper_conf_pldi_malekiyb16_b200.dist import scan_cyclic_virtual

    x = synth.make(n, name, kind, seed=1000 + 37 * k + s + p)
    y = scan_cyclic_virtual(torch.from_numpy(x).cuda(), p, chunk, k, s, incl, lookahead=lookahead)
    torch.cuda.synchronize()
    compare(name, x, y.cpu().numpy(), k, s, incl)


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("k,s", [(1, 1), (2, 1), (4, 4), (8, 1), (3, 5), (8, 8), (6, 3), (7, 2)])
@pytest.mark.parametrize("p", [1, 3, 8])
def test_virtual_ranks_ints(name, k, s, p):
    n = 200_003
    for incl in (True, False):
        _run(name, k, s, n, 7_777, p, incl)


@pytest.mark.parametrize("name,k,s", [("f32", 1, 1), ("f32", 2, 4), ("f64", 1, 3), ("f64", 4, 4)])
@pytest.mark.parametrize("p", [2, 5])
def test_virtual_ranks_floats(name, k, s, p):
    for incl in (True, False):
        _run(name, k, s, 120_001, 9_999, p, incl, kind="small" if k > 1 else "unif01")


@pytest.mark.parametrize("chunk,p,lookahead", [(1, 2, 0), (7, 3, 2), (100_000, 4, 1), (1 << 20, 2, 0),
                                               (333_333, 8, 3)])
def test_chunk_sizes_and_lookahead(chunk, p, lookahead):
    """Chunks of one element, chunks not divisible by s, chunks spanning many tiles, ranks
    without a chunk in the last round, lookahead 0..3."""
    n = 1_000_003 if chunk > 1 else 4_099
    for name, k, s in (("i64", 4, 4), ("i32", 3, 3)):
        _run(name, k, s, n, chunk, p, True, lookahead=lookahead)


@pytest.mark.slow
def test_virtual_ranks_c5_shape():
    """North_star's multi-GPU config shape (int64, order 4, tuple 4) at 2^28 elements over 8
    virtual ranks with the bench's chunk size, element by element against the oracle."""
    from paper_conf_pldi_malekiyb16_b200.dist import scan_cyclic_virtual

    n = 1 << 28
    x = synth.make_torch(n, "i64", "uniform", device="cuda")
    y = scan_cyclic_virtual(x, 8, 1 << 22, 4, 4, True, lookahead=1)
    torch.cuda.synchronize()
    ref = oracle.scan(x.cpu().numpy(), 4, 4, True)[0]
    assert np.array_equal(y.cpu().numpy().view(ref.dtype), ref)


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _worker(rank, world, port, name, k, s, n, chunk, q):
    try:
        import sys

        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        from paper_conf_pldi_malekiyb16_b200.dist import cyclic_chunks, scan_cyclic, to_cyclic

        x = synth.make(n, name, "uniform", seed=5 + k + s)
        xl = to_cyclic(torch.from_numpy(x), chunk, world, rank).cuda()
        st = torch.cuda.Stream()
        ok = True
        for incl in (True, False):
            yt = scan_cyclic(xl, k, s, incl, chunk=chunk, stream=st)  # n from the ranks' lengths
            st.synchronize()
            y = yt.cpu().numpy()
            ref = oracle.scan(x, k, s, incl)[0]
            for g0, ln, lo in cyclic_chunks(n, chunk, world, rank):
                ok &= bool(np.array_equal(y[lo:lo + ln].view(ref.dtype), ref[g0:g0 + ln]))
        q.put((rank, ok, None))
    except Exception:  # pragma: no cover - reported to the parent
        import traceback

        q.put((rank, False, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("name,k,s,n,chunk", [("i64", 4, 4, 1_000_003, 65_536), ("i32", 8, 1, 300_001, 100_000),
                                              ("i32", 2, 3, 77_777, 1_000_000)])
def test_two_rank_scan_cyclic_end_to_end(name, k, s, n, chunk):
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, k, s, n, chunk, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = [q.get(timeout=600) for _ in procs]
    for pr in procs:
        pr.join(timeout=60)
    for rank, ok, err in sorted(res):
        assert ok, f"rank {rank}: {err}"
