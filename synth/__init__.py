"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no prefix sums, no differencing, no
binomials): it only turns (seed, index) into numbers.  Both sides of every parity check draw
their inputs from here, so that the CUDA path and the oracle see bit-identical data.

Generator: counter-based splitmix64.  r_i = mix(seed + (i + 1) * GAMMA) (mod 2^64), i.e. the
i-th output of a splitmix64 stream seeded with `seed`; mix is the splitmix64 output function.
The same formula is implemented twice below -- numpy (host) and torch int64 ops (any device,
used to fill multi-GiB bench/full-size inputs directly in HBM) -- and the two are checked equal
in tests/test_synth.py.

Distributions (SURVEY §8(d) "Value distributions"; the paper only says "32- and 64-bit integer
sequences", and motivates them as delta-decoding residuals "close to zero",
P:172-302):
  uniform : full-range raw bits (exercises wraparound)
  small   : (r mod 17) - 8
  ones    : 1
  pm1int  : (r mod 3) - 1              (floats: exact-in-any-order test)
  unif01  : (r >> 40) * 2^-24 (fp32) / (r >> 11) * 2^-53 (fp64)
"""
from __future__ import annotations

import numpy as np

GAMMA = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
SEED_BASE = 0x53414D00  # "SAM\0"; seed = SEED_BASE + config index

DTYPES = {
    "i32": np.int32,
    "i64": np.int64,
    "f32": np.float32,
    "f64": np.float64,
}
KINDS = ("uniform", "small", "ones", "pm1int", "unif01")

_CHUNK = 1 << 22


def _mix_np(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * np.uint64(M1)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(M2)
    return z ^ (z >> np.uint64(31))


def raw_u64(seed: int, start: int, count: int) -> np.ndarray:
    """r_i for i in [start, start+count) as uint64 (numpy, wraparound)."""
    with np.errstate(over="ignore"):
        i = np.arange(start + 1, start + count + 1, dtype=np.uint64)
        z = np.uint64(seed % (1 << 64)) + i * np.uint64(GAMMA)
        return _mix_np(z)


def _shape(r: np.ndarray, kind: str, dtype: str) -> np.ndarray:
    if kind == "ones":
        return np.ones(r.shape, dtype=DTYPES[dtype])
    if dtype in ("i32", "i64"):
        if kind == "uniform":
            if dtype == "i32":
                return (r & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)
            return r.view(np.int64)
        if kind == "small":
            return ((r % np.uint64(17)).astype(np.int64) - 8).astype(DTYPES[dtype])
        if kind == "pm1int":
            return ((r % np.uint64(3)).astype(np.int64) - 1).astype(DTYPES[dtype])
        raise ValueError(f"kind {kind!r} not defined for {dtype}")
    # floats
    if kind == "unif01":
        if dtype == "f32":
            return ((r >> np.uint64(40)).astype(np.float64) * 2.0**-24).astype(np.float32)
        return (r >> np.uint64(11)).astype(np.float64) * 2.0**-53
    if kind == "pm1int":
        return ((r % np.uint64(3)).astype(np.int64) - 1).astype(DTYPES[dtype])
    if kind == "small":
        return ((r % np.uint64(17)).astype(np.int64) - 8).astype(DTYPES[dtype])
    if kind == "uniform":  # full-range bits would be NaN/Inf soup; use [-1, 1)
        if dtype == "f32":
            return ((r >> np.uint64(40)).astype(np.float64) * 2.0**-23 - 1.0).astype(np.float32)
        return (r >> np.uint64(11)).astype(np.float64) * 2.0**-52 - 1.0
    raise ValueError(f"kind {kind!r} not defined for {dtype}")


def make(n: int, dtype: str, kind: str = "uniform", seed: int = SEED_BASE, start: int = 0) -> np.ndarray:
    """Host array of n values x_{start..start+n-1} (chunked so 2^30 fits in modest RAM)."""
    out = np.empty(n, dtype=DTYPES[dtype])
    for c0 in range(0, n, _CHUNK):
        c1 = min(n, c0 + _CHUNK)
        out[c0:c1] = _shape(raw_u64(seed, start + c0, c1 - c0), kind, dtype)
    return out


# ---------------------------------------------------------------------------------------------
# torch twin (same formula; int64 two's-complement wraparound; logical shifts via masks)
# ---------------------------------------------------------------------------------------------
def _s64(u: int) -> int:
    u %= 1 << 64
    return u - (1 << 64) if u >= 1 << 63 else u


def _lsr(t, r: int):
    return (t >> r) & ((1 << (64 - r)) - 1)


def make_torch(n: int, dtype: str, kind: str = "uniform", seed: int = SEED_BASE, start: int = 0,
               device="cpu", chunk: int = 1 << 26):
    """Same values as make(), generated with torch int64 ops on `device` (e.g. straight into HBM)."""
    import torch

    tdt = {"i32": torch.int32, "i64": torch.int64, "f32": torch.float32, "f64": torch.float64}[dtype]
    out = torch.empty(n, dtype=tdt, device=device)
    if kind == "ones":
        out.fill_(1)
        return out
    g, m1, m2, sd = _s64(GAMMA), _s64(M1), _s64(M2), _s64(seed)
    for c0 in range(0, n, chunk):
        c1 = min(n, c0 + chunk)
        i = torch.arange(start + c0 + 1, start + c1 + 1, dtype=torch.int64, device=device)
        z = i * g + sd
        z = (z ^ _lsr(z, 30)) * m1
        z = (z ^ _lsr(z, 27)) * m2
        r = z ^ _lsr(z, 31)
        out[c0:c1] = _shape_torch(r, kind, dtype, torch)
    return out


def _umod(r, m: int, torch):
    # unsigned r mod m for int64-held uint64 r: (hi*2^32 + lo) mod m
    hi = _lsr(r, 32)
    lo = r & 0xFFFFFFFF
    return ((hi % m) * ((1 << 32) % m) + lo % m) % m


def _shape_torch(r, kind, dtype, torch):
    if dtype in ("i32", "i64"):
        if kind == "uniform":
            if dtype == "i32":
                lo = r & 0xFFFFFFFF
                return torch.where(lo >= (1 << 31), lo - (1 << 32), lo).to(torch.int32)
            return r
        if kind == "small":
            return (_umod(r, 17, torch) - 8).to(r.dtype if dtype == "i64" else torch.int32)
        if kind == "pm1int":
            return (_umod(r, 3, torch) - 1).to(torch.int64 if dtype == "i64" else torch.int32)
        raise ValueError(kind)
    fdt = torch.float32 if dtype == "f32" else torch.float64
    if kind == "unif01":
        if dtype == "f32":
            return (_lsr(r, 40).to(torch.float64) * 2.0**-24).to(fdt)
        return _lsr(r, 11).to(torch.float64) * 2.0**-53
    if kind == "pm1int":
        return (_umod(r, 3, torch) - 1).to(fdt)
    if kind == "small":
        return (_umod(r, 17, torch) - 8).to(fdt)
    if kind == "uniform":
        if dtype == "f32":
            return (_lsr(r, 40).to(torch.float64) * 2.0**-23 - 1.0).to(fdt)
        return _lsr(r, 11).to(torch.float64) * 2.0**-52 - 1.0
    raise ValueError(kind)
