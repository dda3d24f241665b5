"""GPU parity of the delta ENCODER (sam_delta_encode) against the oracle
(oracle.delta: k passes of first-order stride-s differencing), through the C ABI.

Integers bit-exact.  Floats: the kernel evaluates the closed form sum_t (-1)^t C(k,t) x[i-t*s]
 in double and rounds once; the oracle iterates k passes in double (fp32 data) or
x87 long double (fp64 data).  With A_i = sum_t C(k,t)|x[i-t*s]| the two differ by at most
  fp32: 2^-23 |ref| + (k + 2 + k 2^k) 2^-52 A      fp64: (2k + 4) 2^-53 A + k 2^k 2^-64 A
(rounding of the final fp32 store; k+1 double roundings on the GPU side; a pass's error grows by
at most 2x per later pass on the oracle side).  Sizes span several tiles (4096 / 2048 elements)
with ragged tails; misaligned inputs take the scalar staging path.
"""
from __future__ import annotations

import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
import synth
from tests.helpers import DT

pytestmark = pytest.mark.gpu

N_SWEEP = 20011


def S():
    import paper_conf_pldi_malekiyb16_b200 as S

    return S


def gpu_delta(x_np, k, s, offset=0):
    xb = torch.from_numpy(np.concatenate([np.zeros(offset, x_np.dtype), x_np])).cuda()
    x = xb[offset:]
    y = S().delta_encode(x, order=k, tuple=s)
    torch.cuda.synchronize()
    return y.cpu().numpy()


def _abs_weight(x, k, s):
    a = np.abs(x.astype(np.float64))
    A = np.zeros_like(a)
    for t in range(k + 1):
        sh = t * s
        if sh < a.size:
            A[sh:] += math.comb(k, t) * a[: a.size - sh]
    return A


def check(name, x, y, k, s):
    ref = oracle.delta(x, k, s)
    if name in ("i32", "i64"):
        yu = y.view(ref.dtype)
        bad = np.nonzero(yu != ref)[0]
        assert bad.size == 0, f"{name} k={k} s={s} n={x.size}: {bad.size} mismatches, first {bad[:6].tolist()}"
        return
    A = _abs_weight(x, k, s)
    if name == "f32":
        tol = 2.0 ** -23 * np.abs(ref) + (k + 2 + k * 2 ** k) * 2.0 ** -52 * A
        err = np.abs(y.astype(np.float64) - ref)
    else:
        tol = ((2 * k + 4) * 2.0 ** -53 + k * 2 ** k * 2.0 ** -64) * A.astype(np.longdouble)
        err = np.abs(y.astype(np.longdouble) - ref)
    bad = np.nonzero(~(err <= tol))[0]
    assert bad.size == 0, f"{name} k={k} s={s}: {bad.size} outside tolerance, first {bad[:5].tolist()}"


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", range(1, 9))
def test_sweep_dtype_order_tuple(name, k, s):
    x = synth.make(N_SWEEP, name, "uniform", seed=synth.SEED_BASE + 5000 + 10 * k + s)
    check(name, x, gpu_delta(x, k, s), k, s)


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
@pytest.mark.parametrize("n", [1, 2, 7, 63, 64, 65, 2047, 2048, 2049, 4095, 4096, 4097, 3 * 4096, 3 * 4096 + 1])
def test_sizes_and_tile_edges(name, n):
    x = synth.make(n, name, "uniform", seed=n)
    for k, s in ((1, 1), (8, 8), (3, 5)):
        check(name, x, gpu_delta(x, k, s), k, s)


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
def test_misaligned_input_scalar_path(name):
    x = synth.make(40009, name, "uniform", seed=3)
    for k, s in ((1, 1), (2, 3), (8, 8)):
        check(name, x, gpu_delta(x, k, s, offset=1), k, s)


def test_paper_examples():
    x = torch.tensor([1, 2, 3, 4, 5, 2, 4, 6, 8, 10], dtype=torch.int64, device="cuda")
    assert S().delta_encode(x, 1).tolist() == [1, 1, 1, 1, 1, -3, 2, 2, 2, 2]
    assert S().delta_encode(x, 2).tolist() == [1, 0, 0, 0, 0, -4, 5, 0, 0, 0]


def test_empty_and_in_place_refused():
    x = torch.empty(0, dtype=torch.int32, device="cuda")
    assert S().delta_encode(x, 3, 2).numel() == 0
    y = torch.arange(100, dtype=torch.int32, device="cuda")
    with pytest.raises(S().SamError):
        S().delta_encode(y, 1, 1, out=y)


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("k,s", [(1, 1), (2, 1), (4, 4), (8, 8), (3, 7)])
def test_round_trip_encode_then_scan(name, k, s):
    # decode(encode(x)) == x bit for bit, both steps on the GPU
    x = synth.make_torch((1 << 22) + 12345, name, "uniform", seed=k * 10 + s, device="cuda")
    d = S().delta_encode(x, k, s)
    y = S().scan(d, k, s, inclusive=True)
    assert torch.equal(y, x)
    d2 = S().delta_encode(S().scan(x, k, s, inclusive=True), k, s)
    assert torch.equal(d2, x)


@pytest.mark.parametrize("name,k,s", [("i32", 1, 1), ("i32", 8, 8), ("i64", 4, 4), ("f32", 2, 3), ("f64", 3, 2)])
def test_full_size_sampled(name, k, s):
    # 2^30 elements (C2's size) in the bench's launch configuration; sampled outputs, each from the
    # oracle on the window x[i - k s .. i] (out[i] depends on nothing earlier)
    n = 1 << 30 if name in ("i32", "f32") else 1 << 28
    x = synth.make_torch(n, name, "uniform", seed=99, device="cuda")
    y = S().delta_encode(x, k, s)
    torch.cuda.synchronize()
    rng = np.random.default_rng(7)
    idx = np.unique(np.concatenate([rng.integers(0, n, 200), [0, 1, k * s, 4095, 4096, n - 1]]))
    for i in idx.tolist():
        lo = max(0, i - k * s)
        xw = x[lo: i + 1].cpu().numpy()
        yw = np.zeros_like(xw)
        yw[-1] = y[i].item()
        ref = oracle.delta(xw, k, s)
        if name in ("i32", "i64"):
            assert yw.view(ref.dtype)[-1] == ref[-1], f"i={i}"
        else:
            A = _abs_weight(xw, k, s)[-1]
            tol = 2.0 ** -23 * abs(float(ref[-1])) + (k + 2 + k * 2 ** k) * 2.0 ** -52 * A
            assert abs(float(yw[-1]) - float(ref[-1])) <= tol, f"i={i}"
    del x, y
    torch.cuda.empty_cache()


@pytest.mark.parametrize("name", ["i32", "i64", "f32", "f64"])
def test_misaligned_output_scalar_path(name):
    # s = 1 takes the register-window path only when `out` is 16-B aligned; a shifted `out`
    # exercises the scalar stencil on full tiles
    x = synth.make(30011, name, "uniform", seed=4)
    xt = torch.from_numpy(x).cuda()
    buf = torch.empty(x.size + 1, dtype=xt.dtype, device="cuda")
    for k in (1, 5, 8):
        y = S().delta_encode(xt, k, 1, out=buf[1:])
        torch.cuda.synchronize()
        check(name, x, y.cpu().numpy(), k, 1)


@pytest.mark.parametrize("name,k,s,n", [("i32", 3, 5, (1 << 25) * 2 + 12345), ("i64", 8, 8, (1 << 24) + 777),
                                        ("f32", 2, 1, 1000), ("i32", 1, 1, 1)])
def test_host_pipeline(name, k, s, n):
    # sam_delta_encode_host: chunks of 128 MiB (2^25 int32), halos carried across chunks on the device
    x = synth.make_torch(n, name, "uniform", seed=k + s, device="cuda")
    ref = S().delta_encode(x, k, s).cpu()
    xh = x.cpu().pin_memory()
    y = S().delta_encode_host(xh, k, s)
    assert torch.equal(y.view(torch.uint8), ref.view(torch.uint8))
    with pytest.raises(S().SamError):
        S().delta_encode_host(xh, k, s, out=xh)
