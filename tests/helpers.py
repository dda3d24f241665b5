"""Shared test helpers: run the CUDA path through the C ABI and compare with the oracle."""
from __future__ import annotations

import math

import numpy as np

import oracle

DT = {"i32": np.int32, "i64": np.int64, "f32": np.float32, "f64": np.float64}
RTOL = {"f32": 1e-5, "f64": 1e-12}  # north_star tolerance, reading R7


def torch_dtype(name):
    import torch

    return {"i32": torch.int32, "i64": torch.int64, "f32": torch.float32, "f64": torch.float64}[name]


def compare(name: str, x: np.ndarray, y_gpu: np.ndarray, k: int, s: int, inclusive: bool, ref=None,
            exact_float: bool = False):
    """Assert y_gpu matches the oracle: bit-exact for ints (and for floats when exact_float),
    else |y - ref| <= rtol * sqrt(n k) * A with A = oracle scan of |x| (reading R7)."""
    n = x.size
    if ref is None:
        ref = oracle.scan(x, k, s, inclusive)[0]
    if name in ("i32", "i64"):
        yu = y_gpu.view(ref.dtype)
        if not np.array_equal(yu, ref):
            bad = np.nonzero(yu != ref)[0]
            raise AssertionError(f"{name} k={k} s={s} incl={inclusive} n={n}: {bad.size} mismatches, "
                                 f"first at {bad[:8].tolist()} gpu={yu[bad[:4]].tolist()} ref={ref[bad[:4]].tolist()}")
        return
    yg = y_gpu.astype(ref.dtype)
    if exact_float:
        assert np.array_equal(yg, ref), f"{name} k={k} s={s}: integer-valued float result not exact"
        return
    A = oracle.scan(np.abs(x), k, s, inclusive)[0]
    tol = RTOL[name] * math.sqrt(max(1, n) * k) * A
    err = np.abs(yg - ref)
    nan_ok = np.isnan(yg) == np.isnan(ref)
    assert nan_ok.all(), "NaN pattern differs"
    ok = (err <= tol) | np.isnan(ref)
    if not ok.all():
        bad = np.nonzero(~ok)[0]
        raise AssertionError(f"{name} k={k} s={s} incl={inclusive} n={n}: {bad.size} outside tolerance; "
                             f"first {bad[:5].tolist()} err={err[bad[:3]].tolist()} tol={tol[bad[:3]].tolist()}")
