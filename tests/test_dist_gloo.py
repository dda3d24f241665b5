"""Multi-process (world_size 2, gloo, CPU) coverage of the sharded path's host-side logic:
shard offsets from an all-gather of lengths, payload exchange in rank order (the step NCCL
carries on GPUs), and the fold of gathered payloads into each rank's seed -- checked against the
oracle's running state at the shard boundary.  The CUDA kernels themselves are covered by
tests/test_shard_gpu.py (virtual shards on one GPU)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _worker(rank, world, port, k, s, lens, q):
    try:
        import sys

        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        import paper_conf_pldi_malekiyb16_b200 as S
        import synth
        from paper_conf_pldi_malekiyb16_b200.dist import exchange_payloads, shard_offsets

        n = sum(lens)
        x = synth.make(n, "i64", "uniform", seed=77)
        g0, ntot = shard_offsets(lens[rank])
        assert ntot == n and g0 == sum(lens[:rank])
        xl = x[g0:g0 + lens[rank]]
        pb = S.sam_shard_payload_bytes(S.SAM_I64, k, s)
        # this rank's payload (zero-seeded lane states at the shard end), built by the oracle
        pay = np.zeros(pb, dtype=np.uint8)
        hdr = pay[:16].view(np.uint64)
        hdr[0], hdr[1] = lens[rank], g0
        _, run = oracle.scan(xl, k, s, True, phase=g0 % s)
        pay[16:16 + 8 * k * s].view(np.uint64)[:] = run.reshape(k, s).T.reshape(-1)
        gathered = exchange_payloads(torch.from_numpy(pay)).numpy()
        seed = np.zeros(k * s, dtype=np.uint64)
        S.sam_fold_payloads_host(S.SAM_I64, k, s, gathered.ctypes.data, rank, world, seed.ctypes.data)
        _, ref = oracle.scan(x[:g0], k, s, True, phase=0)
        ok = np.array_equal(seed.reshape(s, k), ref.reshape(k, s).T)
        q.put((rank, ok, None))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, False, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("k,s,lens", [(4, 4, [1000, 2333]), (2, 3, [7, 5000]), (8, 1, [4096, 1])])
def test_two_rank_payload_exchange_and_fold(k, s, lens):
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, k, s, lens, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, ok, err in sorted(res):
        assert ok, f"rank {rank}: {err}"
