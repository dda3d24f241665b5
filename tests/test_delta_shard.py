"""Sharded delta encoder (NEXT-2 + §8(e)): the halo exchange's host logic on CPU (pure torch, and
world-size-2/3 gloo process groups), and on the GPU virtual shards through sam_delta_encode_halo
against the whole-array kernel result and the oracle."""
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
from paper_conf_pldi_malekiyb16_b200.dist import TAIL, halo_from_tails, shard_tail

BOUNDS = [
    [0, 5000, 5001, 5003, 9000, 9000, 20011],  # empty shard, 1- and 2-element shards
    [0, 3, 7, 70, 20011],
]


def _halo_oracle_check(x, bounds, k, s):
    """For every shard: oracle.delta(halo ++ shard)[ks:] == oracle.delta(x)[shard]."""
    ks = k * s
    shards = [torch.from_numpy(x[bounds[r]:bounds[r + 1]]) for r in range(len(bounds) - 1)]
    tails = torch.stack([shard_tail(sh) for sh in shards])
    lens = [sh.numel() for sh in shards]
    ref = oracle.delta(x, k, s)
    for r, sh in enumerate(shards):
        h = halo_from_tails(tails, lens, r, ks)
        assert h.numel() == ks
        d = oracle.delta(np.concatenate([h.numpy(), sh.numpy()]), k, s)[ks:]
        assert np.array_equal(d, ref[bounds[r]:bounds[r + 1]]), f"shard {r} k={k} s={s}"


@pytest.mark.parametrize("bounds", BOUNDS)
@pytest.mark.parametrize("k,s", [(1, 1), (3, 2), (8, 8), (2, 7)])
def test_halo_logic_cpu(bounds, k, s):
    x = synth.make(bounds[-1], "i64", "uniform", seed=k + 10 * s)
    _halo_oracle_check(x, bounds, k, s)


def test_tail_width_covers_max_halo():
    assert TAIL >= 8 * 8


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _worker(rank, world, port, lens, k, s, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        n = sum(lens)
        x = synth.make(n, "i32", "uniform", seed=5)
        lo = sum(lens[:rank])
        sh = torch.from_numpy(x[lo:lo + lens[rank]].copy())
        tails = torch.empty(world * TAIL, dtype=sh.dtype)
        dist.all_gather_into_tensor(tails, shard_tail(sh))
        tails = tails.view(world, TAIL)
        lt = torch.empty(world, dtype=torch.int64)
        dist.all_gather_into_tensor(lt, torch.tensor([sh.numel()], dtype=torch.int64))
        h = halo_from_tails(tails, lt.tolist(), rank, k * s)
        d = oracle.delta(np.concatenate([h.numpy(), sh.numpy()]), k, s)[k * s:]
        ok = np.array_equal(d, oracle.delta(x, k, s)[lo:lo + lens[rank]])
        dist.destroy_process_group()
        q.put((rank, ok, ""))
    except Exception as e:  # pragma: no cover
        q.put((rank, False, repr(e)))


@pytest.mark.parametrize("lens,k,s", [([3000, 4001], 2, 3), ([5, 3, 9000], 8, 8)])
def test_halo_exchange_gloo(lens, k, s):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, len(lens), port, lens, k, s, q)) for r in range(len(lens))]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok, _ in res), res


@pytest.mark.gpu
@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
@pytest.mark.parametrize("bounds", BOUNDS + [[0, 1 << 20, (1 << 21) + 3, 3 << 20]])
@pytest.mark.parametrize("k,s", [(1, 1), (4, 1), (3, 5), (8, 8)])
def test_virtual_shards_gpu(name, bounds, k, s):
    import paper_conf_pldi_malekiyb16_b200 as S
    from paper_conf_pldi_malekiyb16_b200.dist import delta_virtual_shards

    x = synth.make_torch(bounds[-1], name, "uniform", seed=k * 7 + s, device="cuda")
    whole = S.delta_encode(x, k, s)
    sharded = delta_virtual_shards(x, bounds, k, s)
    assert torch.equal(whole.view(torch.uint8), sharded.view(torch.uint8))  # bit-identical
    if bounds[-1] <= 20011 and name in ("i32", "i64"):
        ref = oracle.delta(x.cpu().numpy(), k, s)
        assert np.array_equal(sharded.cpu().numpy().view(ref.dtype), ref)


@pytest.mark.gpu
def test_explicit_halo_api():
    import paper_conf_pldi_malekiyb16_b200 as S

    x = torch.tensor([1, 2, 3, 4, 5, 2, 4, 6, 8, 10], dtype=torch.int64, device="cuda")
    # encode x[4:] with the 2 preceding elements as halo == the paper's 2nd-order example tail
    y = S.delta_encode(x[4:].clone(), 2, 1, halo=x[2:4].clone())
    assert y.tolist() == [0, -4, 5, 0, 0, 0]
    with pytest.raises(S.SamError):
        S.delta_encode(x, 2, 1, halo=x[:3].clone())  # wrong halo length
