"""Pins of the oracle's other operators (oracle.scan_op: xor, max, min; SURVEY 8(f) NEXT-4,
P:367-379) against truths independent of its loop: numpy's ufunc accumulate per lane
(the textbook library scan), brute force over prefix sets, the idempotence of max/min (order k =
order 1, exclusive = shift by k lane positions), Lucas' theorem for the order-k xor weights
C(d+k-1, k-1) mod 2, and inversion of order-k xor scans by k-fold xor differencing."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
import synth

DTS = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "f32": np.float32, "f64": np.float64}


def _data(n, name, seed):
    x = synth.make(n, "i64" if name in ("i64", "u64") else "i32", "uniform", seed=seed)
    if name in ("f32", "f64"):
        return (synth.make(n, name, "unif01", seed=seed) * 200 - 100).astype(DTS[name])
    return x.view(np.uint64 if name in ("i64", "u64") else np.uint32).astype(DTS[name], copy=False) \
        if name[0] == "u" else x.astype(DTS[name])


def _lanewise(x, s, fn):
    y = np.empty_like(x)
    for m in range(s):
        y[m::s] = fn(x[m::s])
    return y


def _shift(y, k, s, ident):
    z = np.full_like(y, ident)
    if k * s < y.size:
        z[k * s:] = y[: y.size - k * s]
    return z


@pytest.mark.parametrize("name", list(DTS))
@pytest.mark.parametrize("op", ["max", "min"])
@pytest.mark.parametrize("s", [1, 2, 3, 8])
def test_maxmin_order1_is_numpy_accumulate(name, op, s):
    x = _data(5003, name, seed=s)
    f = {"max": np.fmax, "min": np.fmin}[op] if x.dtype.kind == "f" else {"max": np.maximum, "min": np.minimum}[op]
    ref = _lanewise(x, s, f.accumulate)
    assert np.array_equal(oracle.scan_op(x, op, 1, s, True)[0], ref)
    assert np.array_equal(oracle.scan_op(x, op, 1, s, False)[0], _shift(ref, 1, s, oracle.op_identity(op, x.dtype)))


@pytest.mark.parametrize("name", ["i32", "u64", "f32"])
@pytest.mark.parametrize("op", ["max", "min"])
@pytest.mark.parametrize("k,s", [(2, 1), (5, 3), (8, 8)])
def test_maxmin_idempotent_orders(name, op, k, s):
    """A prefix max of a prefix max is itself: order k inclusive = order 1; k-fold exclusive =
    order-1 inclusive shifted by k lane positions, identity in front."""
    x = _data(4001, name, seed=k * 10 + s)
    f = {"max": np.fmax, "min": np.fmin}[op] if x.dtype.kind == "f" else {"max": np.maximum, "min": np.minimum}[op]
    ref1 = _lanewise(x, s, f.accumulate)
    assert np.array_equal(oracle.scan_op(x, op, k, s, True)[0], ref1)
    assert np.array_equal(oracle.scan_op(x, op, k, s, False)[0], _shift(ref1, k, s, oracle.op_identity(op, x.dtype)))


def test_maxmin_brute_force_and_nan():
    x = np.array([3, -7, 12, 12, -1, 40, 0, 5], dtype=np.int32)
    y = oracle.scan_op(x, "max", 1, 1, True)[0]
    assert y.tolist() == [max(x[: i + 1]) for i in range(x.size)]
    y = oracle.scan_op(x.astype(np.uint32), "min", 1, 2, True)[0]  # unsigned order: -7 is huge
    xu = x.astype(np.uint32)
    assert y.tolist() == [min(xu[i % 2: i + 1: 2]) for i in range(x.size)]
    f = np.array([1.0, np.nan, 0.5, 3.0, np.nan], dtype=np.float64)  # maxNum: NaN operands ignored
    assert oracle.scan_op(f, "max", 1, 1, True)[0].tolist() == [1.0, 1.0, 1.0, 3.0, 3.0]
    # an all-NaN prefix leaves the identity (maxNum ignores NaN operands; the scan is seeded with it)
    assert oracle.scan_op(np.array([np.nan, np.nan]), "min", 1, 1, True)[0].tolist() == [np.inf, np.inf]


@pytest.mark.parametrize("name", ["i32", "u32", "i64", "u64"])
@pytest.mark.parametrize("s", [1, 3, 8])
def test_xor_order1_is_numpy_accumulate(name, s):
    x = _data(5003, name, seed=50 + s)
    ref = _lanewise(x, s, np.bitwise_xor.accumulate)
    assert np.array_equal(oracle.scan_op(x, "xor", 1, s, True)[0], ref)
    assert np.array_equal(oracle.scan_op(x, "xor", 1, s, False)[0], _shift(ref, 1, s, 0))


@pytest.mark.parametrize("k", [1, 2, 3, 4, 7, 8])
@pytest.mark.parametrize("s", [1, 2, 5])
def test_xor_order_k_lucas_brute_force(k, s):
    """Order-k xor scan = sum over GF(2) of C(d+k-1, k-1) x_{i-d s} (d lane positions back), the
    order-k weights reduced mod 2; exclusive weights C(d-1, k-1) (the k-fold shift)."""
    n = 97
    x = _data(n, "u32", seed=k * 7 + s)
    yi = oracle.scan_op(x, "xor", k, s, True)[0]
    ye = oracle.scan_op(x, "xor", k, s, False)[0]
    for i in range(n):
        bi = be = 0
        for d in range(i // s + 1):
            j = i - d * s
            if math.comb(d + k - 1, k - 1) % 2:
                bi ^= int(x[j])
            if d >= 1 and math.comb(d - 1, k - 1) % 2:
                be ^= int(x[j])
        assert int(yi[i]) == bi and int(ye[i]) == be, (i, k, s)


@pytest.mark.parametrize("k,s", [(1, 1), (3, 2), (8, 7)])
def test_xor_inverted_by_k_fold_differencing(k, s):
    x = _data(3001, "u64", seed=k + 100 * s)
    y = oracle.scan_op(x, "xor", k, s, True)[0]
    for _ in range(k):  # x[i] ^= x[i-s], right to left
        y[s:] = y[s:] ^ y[:-s]
    assert np.array_equal(y, x)


def test_xor_streaming_equals_whole():
    x = _data(10007, "i64", seed=3)
    whole = oracle.scan_op(x, "xor", 3, 4, True)[0]
    run = None
    parts = []
    for lo in range(0, x.size, 1234):
        y, run = oracle.scan_op(x[lo:lo + 1234], "xor", 3, 4, True, phase=lo % 4, run=run)
        parts.append(y)
    assert np.array_equal(np.concatenate(parts), whole)
