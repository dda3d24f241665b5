"""Pins for the CPU oracle (oracle/sam_oracle.c) against things other than itself.

Every test here is CPU-only (no "gpu" marker).  Each pins the oracle to a fact fixed by the
paper or by mathematics, chosen so that a plausible mistake (a dropped term, a wrong sign or
index, a transposed operand, a wrong lane, an off-by-one in exclusive) fails at least one:

  golden  : the paper's printed worked examples (tests/golden/*.txt)
  closed  : all-ones -> C(p+k, k) inclusive / C(p, k) exclusive; impulse -> C(p+k-1, k-1)
  brute   : O(n^2) combinatorial sums with Python big ints:
              incl_k[i] = sum_{d>=0} C(d+k-1, k-1) x[i-d*s]   (compositions of d into k parts >= 0)
              excl_k[i] = sum_{d>=k} C(d-1,   k-1) x[i-d*s]   (compositions of d into k parts >= 1)
  inverse : k-th order stride-s differencing (generalises out = in - 2 in_{-1} + in_{-2})
  textbook: de-interleave + numpy.cumsum per lane, k times (the reorder method, P:961-995;
            s = 1 is the conventional prefix sum)
  algebra : composition (order a then b = order a+b), linearity mod 2^w, phase = zero-padding,
            streaming = whole array
  floats  : exact rational arithmetic (fractions.Fraction) on small inputs; integer-valued floats
            equal the integer oracle exactly
"""
from __future__ import annotations

import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
MASK = {np.dtype(np.int32): (1 << 32) - 1, np.dtype(np.int64): (1 << 64) - 1}


def _read_golden(name):
    d = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, val = line.split(":", 1)
            vals = [int(v) for v in val.split()]
            d[key.strip()] = vals if len(vals) > 1 else vals[0]
    return d


def _u(a: np.ndarray) -> list[int]:
    """Python ints of the unsigned reinterpretation."""
    if a.dtype.itemsize == 4:
        return [int(v) for v in np.asarray(a).view(np.uint32)]
    return [int(v) for v in np.asarray(a).view(np.uint64)]


# ----------------------------------------------------------------------------- golden (paper)
@pytest.mark.parametrize("dt", [np.int32, np.int64])
def test_paper_order1_example(dt):
    g = _read_golden("paper_order1_example.txt")
    x = np.array(g["differences"], dtype=dt)
    y = oracle.scan_values(x, k=1, s=1, inclusive=True)
    assert y.tolist() == g["prefix_sum"]
    # the exclusive sum does not include position i
    ye = oracle.scan_values(x, k=1, s=1, inclusive=False)
    assert ye.tolist() == [0] + g["prefix_sum"][:-1]


@pytest.mark.parametrize("dt", [np.int32, np.int64, np.float32, np.float64])
def test_paper_order2_example(dt):
    g = _read_golden("paper_order2_example.txt")
    x = np.array(g["diff2"], dtype=dt)
    y2 = oracle.scan_values(x, k=2, s=1)
    y1 = oracle.scan_values(x, k=1, s=1)
    assert [int(v) for v in y2] == g["values"]
    assert [int(v) for v in y1] == g["diff1"]


# ----------------------------------------------------------------------------- closed forms
@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", range(1, 9))
def test_closed_form_ones_and_impulse(k, s):
    n = 7 * s + 5
    for dt in (np.int32, np.int64):
        mask = MASK[np.dtype(dt)]
        ones = np.ones(n, dtype=dt)
        yi = _u(oracle.scan_values(ones, k, s, True))
        ye = _u(oracle.scan_values(ones, k, s, False))
        assert yi == [math.comb(i // s + k, k) & mask for i in range(n)]
        assert ye == [math.comb(i // s, k) & mask for i in range(n)]
        imp = np.zeros(n, dtype=dt)
        imp[0] = 1
        yimp = _u(oracle.scan_values(imp, k, s, True))
        assert yimp == [(math.comb(i // s + k - 1, k - 1) if i % s == 0 else 0) & mask for i in range(n)]


def test_closed_form_ones_large_k_wraps():
    # order 8 of all-ones over 2^16 elements: C(p+8, 8) overflows 32 bits -> wraparound (R2)
    n = 1 << 16
    x = np.ones(n, dtype=np.int32)
    y = _u(oracle.scan_values(x, 8, 1))
    idx = [0, 1, 1000, 40000, n - 1]
    assert [y[i] for i in idx] == [math.comb(i + 8, 8) % (1 << 32) for i in idx]


# ----------------------------------------------------------------------------- brute force
def _brute(xs: list[int], k: int, s: int, inclusive: bool, mask: int) -> list[int]:
    out = []
    for i in range(len(xs)):
        acc = 0
        for d in range(i // s + 1):
            w = math.comb(d + k - 1, k - 1) if inclusive else (math.comb(d - 1, k - 1) if d >= k else 0)
            acc += w * xs[i - d * s]
        out.append(acc & mask)
    return out


@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("inclusive", [True, False])
def test_brute_force_binomial(k, s, inclusive):
    n = 97
    for dt, name in ((np.int32, "i32"), (np.int64, "i64")):
        x = synth.make(n, name, "uniform", seed=synth.SEED_BASE + 100 + k * 10 + s)
        mask = MASK[np.dtype(dt)]
        xs = [v & mask for v in (int(t) for t in x)]
        assert _u(oracle.scan_values(x, k, s, inclusive)) == _brute(xs, k, s, inclusive, mask)


# ----------------------------------------------------------------------------- inversion
def _kdiff(y: np.ndarray, k: int, s: int) -> np.ndarray:
    """k-th order stride-s difference sum_t (-1)^t C(k,t) y[i-t*s] (missing values are 0)."""
    u = y.view(np.uint64) if y.dtype.itemsize == 8 else y.view(np.uint32)
    out = np.zeros_like(u)
    with np.errstate(over="ignore"):
        for t in range(k + 1):
            c = u.dtype.type(math.comb(k, t) % (1 << (8 * u.dtype.itemsize)))
            sh = np.zeros_like(u)
            if t * s < len(u):
                sh[t * s:] = u[: len(u) - t * s]
            out = out + c * sh if t % 2 == 0 else out - c * sh
    return out.view(y.dtype)


@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", range(1, 9))
def test_inversion_by_kth_order_differencing(k, s):
    for name in ("i32", "i64"):
        x = synth.make(1000 + s, name, "uniform", seed=synth.SEED_BASE + 7 * k + s)
        y = oracle.scan_values(x, k, s, True)
        assert np.array_equal(_kdiff(y, k, s), x)


def test_paper_direct_second_order_formula():
    # out_k = in_k - 2 in_{k-1} + in_{k-2} is the order-2 inverse
    x = synth.make(500, "i64", "small")
    y = oracle.scan_values(x, 2, 1)
    d = y.copy()
    d[1:] -= 2 * y[:-1]
    d[2:] += y[:-2]
    assert np.array_equal(d, x)


# ----------------------------------------------------------------------------- textbook
@pytest.mark.parametrize("k", [1, 2, 3, 8])
@pytest.mark.parametrize("s", range(1, 9))
def test_deinterleave_textbook_cumsum(k, s):
    n = 3001
    for name, ut in (("i32", np.uint32), ("i64", np.uint64)):
        x = synth.make(n, name, "uniform", seed=synth.SEED_BASE + 31 * s + k)
        ref = np.empty(n, dtype=ut)
        for m in range(s):
            lane = x[m::s].view(ut)
            for _ in range(k):
                lane = np.cumsum(lane, dtype=ut)
            ref[m::s] = lane
        assert np.array_equal(oracle.scan(x, k, s, True)[0], ref)


def test_exclusive_is_shift_of_inclusive_by_k_lanes():
    for k in range(1, 9):
        for s in (1, 3, 4):
            x = synth.make(400, "i64", "uniform", seed=k * 100 + s)
            yi = oracle.scan_values(x, k, s, True)
            ye = oracle.scan_values(x, k, s, False)
            assert np.all(ye[: k * s] == 0)
            assert np.array_equal(ye[k * s:], yi[: len(x) - k * s])


# ----------------------------------------------------------------------------- algebra
@pytest.mark.parametrize("a,b", [(1, 1), (1, 3), (2, 5), (4, 4)])
def test_composition(a, b):
    for s in (1, 2, 7):
        x = synth.make(777, "i32", "uniform", seed=a * 13 + b * 7 + s)
        lhs = oracle.scan_values(oracle.scan_values(x, a, s), b, s)
        assert np.array_equal(lhs, oracle.scan_values(x, a + b, s))


def test_linearity_mod_2w():
    x = synth.make(999, "i64", "uniform", seed=1)
    z = synth.make(999, "i64", "uniform", seed=2)
    with np.errstate(over="ignore"):
        lhs = oracle.scan_values(x * np.int64(3) + z, 5, 3)
        rhs = oracle.scan_values(x, 5, 3) * np.int64(3) + oracle.scan_values(z, 5, 3)
    assert np.array_equal(lhs, rhs)


@pytest.mark.parametrize("phase", [0, 1, 3, 6])
def test_phase_equals_zero_padding(phase):
    s, k = 7, 4
    x = synth.make(500, "i64", "uniform", seed=phase)
    padded = np.concatenate([np.zeros(phase, dtype=np.int64), x])
    ref = oracle.scan_values(padded, k, s)[phase:]
    y, _ = oracle.scan(x, k, s, True, phase=phase)
    assert np.array_equal(y.view(np.int64), ref)


@pytest.mark.parametrize("inclusive", [True, False])
def test_streaming_equals_whole(inclusive):
    k, s = 4, 4
    x = synth.make(10007, "i64", "uniform", seed=3)
    whole = oracle.scan_values(x, k, s, inclusive)
    run = None
    parts = []
    pos = 0
    for c in (1, 2, 3, 1000, 17, 5000, 10007):
        c = min(c, len(x) - pos)
        if c <= 0:
            break
        y, run = oracle.scan(x[pos: pos + c], k, s, inclusive, phase=pos % s, run=run)
        parts.append(y.view(np.int64))
        pos += c
    assert pos == len(x)
    assert np.array_equal(np.concatenate(parts), whole)


# ----------------------------------------------------------------------------- floats
def test_long_double_is_x87_extended():
    assert oracle.long_double_bytes() == np.dtype(np.longdouble).itemsize
    assert np.finfo(np.longdouble).nmant >= 63


@pytest.mark.parametrize("dt,name", [(np.float32, "f32"), (np.float64, "f64")])
@pytest.mark.parametrize("k", [1, 2, 4])
def test_float_oracle_against_exact_rationals(dt, name, k):
    s = 3
    x = synth.make(120, name, "unif01", seed=k)
    y = oracle.scan_values(x, k, s, True)
    ex = [Fraction(float(v)) for v in x]
    for _ in range(k):
        run = [Fraction(0)] * s
        for i in range(len(ex)):
            run[i % s] += ex[i]
            ex[i] = run[i % s]
    eps = 2.0**-50 if dt == np.float32 else 2.0**-60   # double / long double accumulation
    for i in range(len(ex)):
        ref = ex[i]
        assert abs(Fraction(float(y[i]) if dt == np.float32 else Fraction(str(y[i]))) - ref) <= eps * len(x) * k * abs(ref) + 1e-300


@pytest.mark.parametrize("name,iname", [("f32", "i32"), ("f64", "i64")])
def test_integer_valued_floats_exact(name, iname):
    x = synth.make(5000, name, "pm1int", seed=5)
    xi = synth.make(5000, iname, "pm1int", seed=5)
    for k in (1, 2, 3):
        yf = oracle.scan_values(x, k, 2)
        yi = oracle.scan_values(xi, k, 2)
        assert np.array_equal(yf.astype(np.float64), yi.astype(np.float64))


def test_oracle_rejects_bad_args():
    with pytest.raises(ValueError):
        oracle.scan(np.zeros(4, np.int32), 1, 2, True, phase=2)
    with pytest.raises(ValueError):
        oracle.scan(np.zeros(4, np.int32), 0, 1, True)


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("k,s", [(1, 1), (3, 1), (2, 5), (8, 8), (4, 3)])
def test_allcores_context_scan_matches_serial_oracle(name, k, s):
    """bench.py's all-cores CPU context number runs oracle.scan_allcores (k passes of two-phase
    order-1 scans over chunks); it must equal the serial oracle bit for bit, for chunk counts that
    do and do not divide n or s."""
    x = synth.make(100_003, name, "uniform", seed=k * 10 + s)
    ref = oracle.scan(x, k, s, True)[0]
    for threads in (1, 3, 8):
        got = oracle.scan_allcores(x, k, s, threads=threads)
        assert np.array_equal(got, ref), f"threads={threads}"
