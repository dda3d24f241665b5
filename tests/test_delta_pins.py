"""Pins for the oracle's delta ENCODER (oracle.delta, sam_oracle.c oracle_delta_*), SURVEY 8(f)
NEXT-2: the k-th order, stride-s difference sequence.

Every test is CPU-only.  A plausible mistake (left-to-right instead of right-to-left passes, a
wrong stride, a dropped pass, a sign error, a non-zero "missing" value) fails at least one:

  golden  : the paper's printed examples: 1st-order differences and the 2nd-order
            difference sequence, both direct and as diff-of-diffs
  direct  : the paper's closed form generalised, out_i = sum_t (-1)^t C(k,t) in_{i-t*s}
            (out_k = in_k - 2 in_{k-1} + in_{k-2}), Python big ints, missing = 0
  inverse : the order-k inclusive prefix sum (pinned independently in test_oracle_pins.py)
            decodes the order-k difference sequence and vice versa
  poly    : k-th differences annihilate polynomials of degree < k in the lane position and
            map m^k to the constant k! (textbook finite differences), after the first k*s items
  floats  : exact rationals; integer-valued floats equal the integer oracle
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
MASK = {4: (1 << 32) - 1, 8: (1 << 64) - 1}


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


def _signed(a):
    return [int(v) for v in np.asarray(a).view(np.int32 if a.dtype.itemsize == 4 else np.int64)]


@pytest.mark.parametrize("dt", [np.int32, np.int64, np.float32, np.float64])
def test_paper_examples(dt):
    g1 = _read_golden("paper_order1_example.txt")
    g2 = _read_golden("paper_order2_example.txt")
    x = np.array(g1["prefix_sum"], dtype=dt)
    d1 = oracle.delta(x, 1, 1)
    assert [int(v) for v in (d1 if dt in (np.float32, np.float64) else _signed(d1))] == g1["differences"]
    v = np.array(g2["values"], dtype=dt)
    for k, key in ((1, "diff1"), (2, "diff2")):
        d = oracle.delta(v, k, 1)
        got = [int(e) for e in d] if dt in (np.float32, np.float64) else _signed(d)
        assert got == g2[key]


def _direct(xs, k, s, mask):
    return [sum((-1) ** t * math.comb(k, t) * xs[i - t * s] for t in range(k + 1) if i - t * s >= 0) & mask
            for i in range(len(xs))]


@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", [1, 2, 3, 5, 8])
def test_direct_binomial_form(k, s):
    for name in ("i32", "i64"):
        x = synth.make(6 * s * k + 7, name, "uniform", seed=100 * k + s)
        w = x.dtype.itemsize
        xs = [int(v) for v in x.view(np.uint32 if w == 4 else np.uint64)]
        got = [int(v) for v in oracle.delta(x, k, s)]
        assert got == _direct(xs, k, s, MASK[w])


@pytest.mark.parametrize("k", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("s", [1, 2, 4, 7, 8])
@pytest.mark.parametrize("name", ["i32", "i64"])
def test_inverse_of_inclusive_scan(k, s, name):
    x = synth.make(3000 + s, name, "uniform", seed=k * 31 + s)
    d = oracle.delta(x, k, s).view(x.dtype)
    assert np.array_equal(oracle.scan_values(d, k, s, True), x)
    y = oracle.scan_values(x, k, s, True)
    assert np.array_equal(oracle.delta(y, k, s).view(x.dtype), x)


@pytest.mark.parametrize("k", range(1, 9))
@pytest.mark.parametrize("s", [1, 3, 8])
def test_polynomials(k, s):
    n = 12 * s + 40
    m = np.arange(n) // s + 3  # lane position (shifted so no factor is 0)
    rng = np.random.default_rng(k * 10 + s)
    coef = rng.integers(-50, 50, size=k)
    low = sum(int(c) * m.astype(object) ** j for j, c in enumerate(coef))  # degree < k
    x = np.array([int(v) for v in low], dtype=np.int64)
    d = oracle.delta(x, k, s).view(np.int64)
    assert (d[k * s:] == 0).all()
    x = np.array([int(v) ** k for v in m], dtype=np.int64)
    d = oracle.delta(x, k, s).view(np.int64)
    assert (d[k * s:] == math.factorial(k)).all()


@pytest.mark.parametrize("name,dt", [("f32", np.float32), ("f64", np.float64)])
@pytest.mark.parametrize("k", [1, 3, 6])
def test_float_against_exact_rationals(name, dt, k):
    s = 2
    x = synth.make(60, name, "uniform", seed=k)
    d = oracle.delta(x, k, s)
    xs = [Fraction(float(v)) for v in x]
    exact = [sum((-1) ** t * math.comb(k, t) * xs[i - t * s] for t in range(k + 1) if i - t * s >= 0)
             for i in range(x.size)]
    for e, g, i in zip(exact, d, range(x.size)):
        A = sum(math.comb(k, t) * abs(xs[i - t * s]) for t in range(k + 1) if i - t * s >= 0)
        eps = 2.0 ** -52 if name == "f32" else 2.0 ** -63  # accumulator precision (double / x87)
        # pass p's rounding error is amplified by at most 2^(k-p) by the later passes
        assert abs(Fraction(*g.as_integer_ratio()) - e) <= k * 2 ** k * eps * A


def test_integer_valued_floats_equal_int_oracle():
    x = synth.make(777, "i32", "uniform", seed=5) % 1000
    for dt in (np.float32, np.float64):
        d = oracle.delta(x.astype(dt), 4, 3)
        assert [int(v) for v in d] == _signed(oracle.delta(x.astype(np.int64), 4, 3))


def test_empty_and_short():
    for n in range(0, 5):
        x = np.arange(1, n + 1, dtype=np.int64)
        assert _signed(oracle.delta(x, 3, 8)) == list(range(1, n + 1))  # i < s: nothing s back
