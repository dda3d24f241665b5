"""Block-cyclic multi-GPU path, host side, no GPU: the chunk layout, and the
round fold sam_cyclic_fold_host (the template the device kernel runs) chained over rounds --
checked against the ORACLE's streamed running state before every chunk, alone and across two gloo
processes exchanging their payloads (the step NCCL carries on GPUs).  Payloads are built by the
oracle (zero-seeded lane states at each chunk's end), so nothing here comes from the CUDA path."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_pldi_malekiyb16_b200.dist import (cyclic_chunks, cyclic_local_len, cyclic_rounds, from_cyclic,
                                                   to_cyclic)

DC = {"i32": 0, "i64": 1, "f32": 2, "f64": 3}
UT = {"i32": np.uint32, "i64": np.uint64, "f32": np.float32, "f64": np.float64}


@pytest.mark.parametrize("n,chunk,p", [(0, 4, 2), (1, 4, 2), (8, 4, 2), (9, 4, 2), (100, 7, 3), (1000, 1, 8),
                                       (1000, 999, 8), (12345, 100, 5)])
def test_layout_covers_every_element_once(n, chunk, p):
    seen = np.zeros(n, dtype=np.int64)
    rounds = cyclic_rounds(n, chunk, p)
    for g in range(p):
        ch = cyclic_chunks(n, chunk, p, g)
        assert len(ch) <= rounds
        lo = 0
        for r, (g0, ln, l0) in enumerate(ch):
            assert g0 == (r * p + g) * chunk and l0 == lo and 0 < ln <= chunk
            seen[g0:g0 + ln] += 1
            lo += ln
        assert lo == cyclic_local_len(n, chunk, p, g)
    assert (seen == 1).all()
    if n:
        assert max(len(cyclic_chunks(n, chunk, p, g)) for g in range(p)) == rounds
    x = torch.arange(n, dtype=torch.int64)
    parts = [to_cyclic(x, chunk, p, g) for g in range(p)]
    if n:
        assert torch.equal(from_cyclic(parts, chunk, n), x)


def _payload(S, name, x, g0, ln, k, s):
    """Oracle-built payload of the chunk x[g0:g0+ln]: [n][g][lane states at the chunk end]."""
    pb = S.sam_shard_payload_bytes(DC[name], k, s)
    buf = np.zeros(pb, dtype=np.uint8)
    hdr = buf[:16].view(np.uint64)
    hdr[0], hdr[1] = ln, g0
    if ln:
        _, run = oracle.scan(x[g0:g0 + ln], k, s, True, phase=g0 % s)
        st = run.reshape(k, s).T.reshape(-1)
        w = np.dtype(UT[name]).itemsize
        if name.startswith("i"):
            buf[16:16 + k * s * w].view(UT[name])[:] = st.view(UT[name])
        else:
            buf[16:16 + k * s * w].view(UT[name])[:] = st.astype(UT[name])
    return buf


def _state_before(x, g0, k, s, name):
    _, run = oracle.scan(x[:g0], k, s, True, phase=0)
    st = run.reshape(k, s).T
    return st.view(UT[name]) if name.startswith("i") else st.astype(np.float64)


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("k,s,n,chunk,p", [(1, 1, 1000, 64, 4), (4, 4, 5003, 333, 3), (8, 8, 4001, 250, 2),
                                           (3, 5, 2999, 101, 8), (2, 7, 777, 1000, 4), (5, 3, 1234, 17, 5)])
def test_round_fold_chain_matches_oracle(name, k, s, n, chunk, p):
    """seed(r, g) = base_r (+) payloads of round r, ranks < g; base_{r+1} = base_r (+) all p --
    equals the oracle's running state before chunk r*p+g, for every round and rank (empty
    payloads for ranks with no chunk in the last round, chunk lengths not divisible by s)."""
    import paper_conf_pldi_malekiyb16_b200 as S
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    x = synth.make(n, name, "uniform", seed=k * 100 + s)
    R = cyclic_rounds(n, chunk, p)
    base = np.zeros(k * s, dtype=UT[name])
    for r in range(R):
        pays = []
        for g in range(p):
            c = r * p + g
            g0 = c * chunk
            ln = max(0, min(chunk, n - g0))
            pays.append(_payload(S, name, x, g0, ln, k, s))
        buf = np.concatenate(pays)
        newbase = np.zeros_like(base)
        for g in range(p):
            seed = np.zeros_like(base)
            S.sam_cyclic_fold_host(DC[name], k, s, buf.ctypes.data, g, p, base.ctypes.data, seed.ctypes.data,
                                   newbase.ctypes.data if g == 0 else None)
            g0 = min((r * p + g) * chunk, n)
            assert np.array_equal(seed.reshape(s, k), _state_before(x, g0, k, s, name)), f"round {r} rank {g}"
        base = newbase
    assert np.array_equal(base.reshape(s, k), _state_before(x, n, k, s, name))


def test_round_fold_floats_close():
    import paper_conf_pldi_malekiyb16_b200 as S
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    name, k, s, n, chunk, p = "f64", 3, 2, 4001, 300, 3
    x = synth.make(n, name, "unif01", seed=5)
    base = np.zeros(k * s)
    for r in range(cyclic_rounds(n, chunk, p)):
        buf = np.concatenate([_payload(S, name, x, (r * p + g) * chunk, max(0, min(chunk, n - (r * p + g) * chunk)), k, s)
                              for g in range(p)])
        nb = np.zeros_like(base)
        for g in range(p):
            seed = np.zeros_like(base)
            S.sam_cyclic_fold_host(DC[name], k, s, buf.ctypes.data, g, p, base.ctypes.data, seed.ctypes.data,
                                   nb.ctypes.data)
            ref = _state_before(x, min((r * p + g) * chunk, n), k, s, name)
            assert np.allclose(seed.reshape(s, k), ref, rtol=1e-12, atol=0)
        base = nb


def test_cyclic_fold_validates_arguments():
    import paper_conf_pldi_malekiyb16_b200 as S
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    L = S.lib()
    buf = (ctypes_buf := np.zeros(4096, dtype=np.uint8)).ctypes.data
    assert L.sam_cyclic_fold(1, 9, 1, buf, 0, 1, None, buf, None, None) == -2      # order 9
    assert L.sam_cyclic_fold(1, 1, 1, buf, 2, 2, None, buf, None, None) == -1      # rank >= nranks
    assert L.sam_cyclic_fold(1, 1, 1, None, 0, 1, None, buf, None, None) == -1     # null payloads
    assert L.sam_cyclic_fold_host(1, 1, 1, buf, 0, 1, None, None, None) == -1     # null seed
    assert ctypes_buf.size == 4096


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _worker(rank, world, port, k, s, n, chunk, q):
    try:
        import sys

        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_pldi_malekiyb16_b200 as S
        from paper_conf_pldi_malekiyb16_b200.dist import exchange_payloads

        x = synth.make(n, "i64", "uniform", seed=91)
        base = np.zeros(k * s, dtype=np.uint64)
        ok = True
        for r in range(cyclic_rounds(n, chunk, world)):
            g0 = (r * world + rank) * chunk
            pay = _payload(S, "i64", x, g0, max(0, min(chunk, n - g0)), k, s)
            gathered = exchange_payloads(torch.from_numpy(pay)).numpy()
            seed = np.zeros_like(base)
            S.sam_cyclic_fold_host(1, k, s, gathered.ctypes.data, rank, world, base.ctypes.data, seed.ctypes.data,
                                   base.ctypes.data)
            ok &= bool(np.array_equal(seed.reshape(s, k), _state_before(x, min(g0, n), k, s, "i64")))
        ok &= bool(np.array_equal(base.reshape(s, k), _state_before(x, n, k, s, "i64")))
        q.put((rank, ok, None))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, False, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("k,s,n,chunk", [(4, 4, 5003, 300), (8, 1, 999, 1000), (2, 3, 4000, 77)])
def test_two_rank_round_exchange_and_fold(k, s, n, chunk):
    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, k, s, n, chunk, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = [q.get(timeout=240) for _ in procs]
    for pr in procs:
        pr.join(timeout=60)
    for rank, ok, err in sorted(res):
        assert ok, f"rank {rank}: {err}"
