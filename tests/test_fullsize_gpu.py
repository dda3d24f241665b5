"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (one sam_scan
launch over inputs resident in HBM), compared with the CPU oracle element by element:
  C2  n = 2^30 int32, order 1, tuple 1
  C3  n = 2^28 int32 / int64, orders 1..8 (subset), tuple 1
  C4  n = 2^28 int64 tuples s = 2..8 at orders 1, 2; fp32 / fp64 order 1 tuples (exact on
      integer-valued inputs, tolerance on unif01, R7)
  C5  int64 order 4 tuple 4: 8 uneven virtual shards (state pass, payload fold, seeded scans) equal
      the unsharded scan bit for bit at 2^30, and the oracle at 2^28
"""
from __future__ import annotations

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
import synth
from tests.helpers import compare

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def _scan(x, k, s, incl):
    import paper_conf_pldi_malekiyb16_b200 as S

    y = S.scan(x, k, s, incl)
    torch.cuda.synchronize()
    return y


def _check_int(name, n, k, s, incl=True, seed=1):
    x = synth.make_torch(n, name, "uniform", seed=synth.SEED_BASE + seed, device="cuda")
    y = _scan(x, k, s, incl).cpu().numpy()
    xh = x.cpu().numpy()
    del x
    torch.cuda.empty_cache()
    ref = oracle.scan(xh, k, s, incl)[0]
    assert np.array_equal(y.view(ref.dtype), ref), f"{name} n={n} k={k} s={s} incl={incl}"


def test_C2_int32_2p30_order1():
    _check_int("i32", 1 << 30, 1, 1, True, seed=1)


@pytest.mark.parametrize("k", [1, 2, 3, 4, 8])
def test_C3_int32_2p28_orders(k):
    _check_int("i32", 1 << 28, k, 1, True, seed=2)


@pytest.mark.parametrize("k", [1, 2, 5, 8])
def test_C3_int64_2p28_orders(k):
    _check_int("i64", 1 << 28, k, 1, True, seed=3)


def test_C3_exclusive_spot():
    _check_int("i32", 1 << 28, 4, 1, False, seed=4)


@pytest.mark.parametrize("s", [2, 3, 5, 8])
@pytest.mark.parametrize("k", [1, 2])
def test_C4_int64_2p28_tuples(k, s):
    _check_int("i64", 1 << 28, k, s, True, seed=5)


@pytest.mark.parametrize("name", ["f32", "f64"])
@pytest.mark.parametrize("s", [1, 3, 8])
def test_C4_float_tuples(name, s):
    n = 1 << 28
    # integer-valued +-1 random walk: partial sums stay < 2^15, exact in any association order
    x = synth.make_torch(n, name, "pm1int", seed=synth.SEED_BASE + 6, device="cuda")
    y = _scan(x, 1, s, True).cpu().numpy()
    xh = x.cpu().numpy()
    compare(name, xh, y, 1, s, True, exact_float=True)
    # unif01: tolerance rtol*sqrt(n k)*A on a 2^24 prefix (oracle cost bound)
    m = 1 << 24
    x = synth.make_torch(m, name, "unif01", seed=synth.SEED_BASE + 7, device="cuda")
    y = _scan(x, 1, s, True).cpu().numpy()
    compare(name, x.cpu().numpy(), y, 1, s, True)


def test_C5_sharded_order4_tuple4():
    from paper_conf_pldi_malekiyb16_b200.dist import scan_virtual_shards

    k, s = 4, 4
    for n, with_oracle in ((1 << 28, True), (1 << 30, False)):
        x = synth.make_torch(n, "i64", "uniform", seed=synth.SEED_BASE + 8, device="cuda")
        rng = np.random.default_rng(5)
        cuts = sorted(set(int(c) for c in rng.integers(1, n, size=7)))
        bounds = [0] + cuts + [n]
        ys = scan_virtual_shards(x, bounds, k, s, True)
        y1 = _scan(x, k, s, True)
        assert torch.equal(ys, y1)
        if with_oracle:
            ref = oracle.scan(x.cpu().numpy(), k, s, True)[0]
            assert np.array_equal(ys.cpu().numpy().view(ref.dtype), ref)
        del x, ys, y1
        torch.cuda.empty_cache()


def test_C5_2p33_int64_order4_tuple4_single_gpu():
    """n = 2^33 > 2^32 elements (C5 strong at p = 1): 64 GiB in + 64 GiB
    out in HBM, one launch.  Verified against the chunked oracle (the same serial loop with its
    per-(pass, lane) running sums carried across chunks) on D2H chunks of the output."""
    import paper_conf_pldi_malekiyb16_b200 as S

    free, _ = torch.cuda.mem_get_info()
    n = 1 << 33
    if free < 2 * 8 * n + (4 << 30):
        pytest.skip(f"needs ~132 GiB free HBM, have {free / 2**30:.0f} GiB")
    k, s = 4, 4
    x = synth.make_torch(n, "i64", "uniform", seed=synth.SEED_BASE + 9, device="cuda")
    y = torch.empty_like(x)
    S.scan(x, k, s, True, out=y)
    torch.cuda.synchronize()
    run = None
    chunk = 1 << 28
    for off in range(0, n, chunk):
        xc = x[off:off + chunk].cpu().numpy()
        ref, run = oracle.scan(xc, k, s, True, phase=off % s, run=run)
        got = y[off:off + chunk].cpu().numpy().view(ref.dtype)
        assert np.array_equal(got, ref), f"mismatch in chunk at {off}"
    # the state-pass reduction kernel (sam_shard_state) over the same 2^33 elements: the zero-seeded
    # state of every lane at its last element = the chunked oracle's final running sums
    import ctypes

    pay = torch.zeros(S.sam_shard_payload_bytes(S.SAM_I64, k, s), dtype=torch.uint8, device="cuda")
    S.sam_shard_state(S.SAM_I64, k, s, ctypes.c_void_p(x.data_ptr()), n, 0, ctypes.c_void_p(pay.data_ptr()))
    torch.cuda.synchronize()
    st = pay.cpu().numpy()[16:16 + 8 * k * s].view(np.uint64).reshape(s, k)
    assert np.array_equal(st, np.asarray(run).reshape(k, s).T.view(np.uint64)), "state pass at 2^33"

