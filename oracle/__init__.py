"""ORACLE -- TEST INFRASTRUCTURE ONLY (see sam_oracle.c for the citations and the contract).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package.  The product package (paper_conf_pldi_malekiyb16_b200) never imports it
and it never imports the product package.

scan(x, k, s, inclusive, phase=0, run=None) -> (y, run)
delta(x, k, s) -> d       k-th order stride-s difference sequence (the encoder);
                          same result dtypes as scan
    x      : 1-D numpy array, dtype int32 / int64 / float32 / float64
    y      : uint32 / uint64 (reinterpret as int32/int64 for comparisons), float64 for fp32
             data, np.longdouble for fp64 data
    phase  : lane of x[0] (global index mod s)
    run    : per-(pass, lane) running sums, k*s entries (accumulator dtype); pass the returned
             `run` back in to continue a stream (chunk-outer nesting of the same loop).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sam_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None
_SRC_MT = os.path.join(_HERE, "cpu_allcores.c")
_LIB_MT = os.path.join(_HERE, "liboracle_mt.so")
_lib_mt = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C, IEEE semantics: no fast-math, no contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off",
                               "-fno-fast-math", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def build_allcores(force: bool = False) -> str:
    """Compile the all-cores CPU context scan (OpenMP; cpu_allcores.c)."""
    if force or not os.path.exists(_LIB_MT) or os.path.getmtime(_LIB_MT) < os.path.getmtime(_SRC_MT):
        tmp = _LIB_MT + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-std=c11", "-fPIC", "-shared", "-fopenmp", "-o", tmp, _SRC_MT])
        os.replace(tmp, _LIB_MT)
    return _LIB_MT


def scan_allcores(x: np.ndarray, k: int, s: int = 1, phase: int = 0, threads: int | None = None) -> np.ndarray:
    """All-cores CPU context scan (inclusive, integers only): k passes of two-phase order-1 scans
    over `threads` chunks (default: os.cpu_count()).  Returns uint32/uint64 like scan()."""
    global _lib_mt
    if _lib_mt is None:
        L = ctypes.CDLL(build_allcores())
        for name in ("allcores_scan_u32", "allcores_scan_u64"):
            fn = getattr(L, name)
            fn.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int]
            fn.restype = ctypes.c_int
        _lib_mt = L
    x = np.ascontiguousarray(x)
    if x.dtype.kind not in "iu":
        raise ValueError("scan_allcores: integer data only")
    acc = np.uint32 if x.dtype.itemsize == 4 else np.uint64
    a = x.view(acc).copy()
    nt = int(threads or os.cpu_count() or 1)
    fn = _lib_mt.allcores_scan_u32 if acc is np.uint32 else _lib_mt.allcores_scan_u64
    rc = fn(a.ctypes.data, a.size, int(k), int(s), int(phase), nt)
    if rc != 0:
        raise ValueError(f"allcores scan rejected arguments (rc={rc})")
    return a


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        P = ctypes.c_void_p
        for name in ("oracle_scan_u32", "oracle_scan_u64", "oracle_scan_f64acc", "oracle_scan_ldacc"):
            fn = getattr(lib, name)
            fn.argtypes = [P, ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, P]
            fn.restype = ctypes.c_int
        for name in ("oracle_delta_u32", "oracle_delta_u64", "oracle_delta_f64acc", "oracle_delta_ldacc"):
            fn = getattr(lib, name)
            fn.argtypes = [P, ctypes.c_uint64, ctypes.c_int, ctypes.c_int]
            fn.restype = ctypes.c_int
        for name in ("oracle_scan_op_i32", "oracle_scan_op_u32", "oracle_scan_op_i64", "oracle_scan_op_u64",
                     "oracle_scan_op_f32", "oracle_scan_op_f64"):
            fn = getattr(lib, name)
            fn.argtypes = [P, ctypes.c_uint64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, P]
            fn.restype = ctypes.c_int
        lib.oracle_sizeof_long_double.restype = ctypes.c_int
        _lib = lib
    return _lib


_ACC = {
    np.dtype(np.int32): (np.uint32, "oracle_scan_u32"),
    np.dtype(np.uint32): (np.uint32, "oracle_scan_u32"),
    np.dtype(np.int64): (np.uint64, "oracle_scan_u64"),
    np.dtype(np.uint64): (np.uint64, "oracle_scan_u64"),
    np.dtype(np.float32): (np.float64, "oracle_scan_f64acc"),
    np.dtype(np.float64): (np.longdouble, "oracle_scan_ldacc"),
}


def acc_dtype(dtype) -> np.dtype:
    return np.dtype(_ACC[np.dtype(dtype)][0])


def scan(x: np.ndarray, k: int, s: int = 1, inclusive: bool = True, phase: int = 0, run=None):
    lib = _load()
    x = np.ascontiguousarray(x)
    acc, fname = _ACC[x.dtype]
    if x.dtype.kind in "iu":
        a = x.view(acc).copy() if x.dtype.itemsize == np.dtype(acc).itemsize else x.astype(acc)
    else:
        a = x.astype(acc)
    if run is None:
        run = np.zeros(k * s, dtype=acc)
    else:
        run = np.ascontiguousarray(run, dtype=acc)
        assert run.size == k * s
    rc = getattr(lib, fname)(a.ctypes.data, a.size, int(k), int(s), int(bool(inclusive)), int(phase),
                             run.ctypes.data)
    if rc != 0:
        raise ValueError(f"oracle rejected arguments (rc={rc}): k={k} s={s} phase={phase}")
    return a, run


def scan_values(x: np.ndarray, k: int, s: int = 1, inclusive: bool = True) -> np.ndarray:
    """Convenience: result reinterpreted in the input's signedness for ints."""
    y, _ = scan(x, k, s, inclusive)
    if x.dtype.kind in "iu":
        return y.view(x.dtype)
    return y


def delta(x: np.ndarray, k: int, s: int = 1) -> np.ndarray:
    """k-th order stride-s difference sequence of x (k passes of first-order differencing,
    missing values zero; sam_oracle.c oracle_delta_*).  Ints: uint32/uint64 result."""
    lib = _load()
    x = np.ascontiguousarray(x)
    acc, fname = _ACC[x.dtype]
    fname = fname.replace("oracle_scan_", "oracle_delta_")
    if x.dtype.kind in "iu":
        a = x.view(acc).copy() if x.dtype.itemsize == np.dtype(acc).itemsize else x.astype(acc)
    else:
        a = x.astype(acc)
    rc = getattr(lib, fname)(a.ctypes.data, a.size, int(k), int(s))
    if rc != 0:
        raise ValueError(f"oracle rejected arguments (rc={rc}): k={k} s={s}")
    return a


OPS = {"add": 0, "xor": 1, "max": 2, "min": 3}
_OP_FN = {np.dtype(np.int32): "i32", np.dtype(np.uint32): "u32", np.dtype(np.int64): "i64",
          np.dtype(np.uint64): "u64", np.dtype(np.float32): "f32", np.dtype(np.float64): "f64"}


def op_identity(op: str, dtype):
    """Identity element of `op` on dtype (reading R14): xor 0; max: lowest value (-inf for
    floats); min: highest value (+inf for floats)."""
    dt = np.dtype(dtype)
    if op == "xor":
        return dt.type(0)
    if dt.kind == "f":
        return dt.type(-np.inf if op == "max" else np.inf)
    info = np.iinfo(dt)
    return dt.type(info.min if op == "max" else info.max)


def scan_op(x: np.ndarray, op: str, k: int, s: int = 1, inclusive: bool = True, phase: int = 0, run=None):
    """Order-k, tuple-s scan of x under `op` in {"xor", "max", "min"} (sam_oracle.c
    oracle_scan_op_*): the serial loop with op in place of +, in the element type.  Returns (y, run).
    ("add" is scan().)"""
    lib = _load()
    x = np.ascontiguousarray(x)
    if op not in ("xor", "max", "min"):
        raise ValueError("scan_op: op must be xor, max or min (add is oracle.scan)")
    if op == "xor" and x.dtype.kind == "f":
        raise ValueError("xor is defined for integers only")
    a = x.copy()
    if run is None:
        run = np.full(k * s, op_identity(op, x.dtype), dtype=x.dtype)
    else:
        run = np.ascontiguousarray(run, dtype=x.dtype)
    fn = getattr(lib, "oracle_scan_op_" + _OP_FN[x.dtype])
    rc = fn(a.ctypes.data, a.size, OPS[op], int(k), int(s), int(bool(inclusive)), int(phase), run.ctypes.data)
    if rc != 0:
        raise ValueError(f"oracle rejected arguments (rc={rc})")
    return a, run


def long_double_bytes() -> int:
    return _load().oracle_sizeof_long_double()
