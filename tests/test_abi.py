"""C-ABI boundary checks that need no GPU: libsam.so loads, exports every symbol include/sam.h
declares, validates arguments synchronously (before any CUDA call), and its host fold (the same
template the device fold kernel runs) matches the oracle's streamed state."""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "sam.h")


def _lib():
    import paper_conf_pldi_malekiyb16_b200 as S

    from paper_conf_pldi_malekiyb16_b200 import _build

    _build.build()
    return S


def declared_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(sam_[a-z_]+)\s*\(", txt)))


def test_header_declares_the_north_star_entry_points():
    syms = declared_symbols()
    for s in ("sam_scan", "sam_shard_state", "sam_shard_scan", "sam_shard_payload_bytes", "sam_last_error"):
        assert s in syms


def test_library_exports_every_declared_symbol():
    S = _lib()
    L = ctypes.CDLL(S.LIB_PATH)
    missing = [s for s in declared_symbols() if not hasattr(L, s)]
    assert not missing, f"libsam.so lacks {missing}"


def test_library_is_sm100a_only():
    # the cubin inside libsam.so targets sm_100a (cuobjdump lists the embedded ELF arch)
    import subprocess

    S = _lib()
    out = subprocess.run(["cuobjdump", "--list-elf", S.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out and "sm_90" not in out


@pytest.mark.parametrize("order,tuple_,code", [(0, 1, -2), (9, 1, -2), (1, 0, -2), (1, 9, -2)])
def test_validation_unsupported(order, tuple_, code):
    S = _lib()
    L = S.lib()
    x = (ctypes.c_int * 4)()
    assert L.sam_scan(0, order, tuple_, 1, ctypes.addressof(x), ctypes.addressof(x), 4, None) == code
    assert "1..8" in S.sam_last_error()


def test_validation_invalid_args():
    S = _lib()
    L = S.lib()
    buf = (ctypes.c_int64 * 64)()
    base = ctypes.addressof(buf)
    assert L.sam_scan(7, 1, 1, 1, base, base, 4, None) == -2                    # unknown dtype
    assert L.sam_scan(0, 1, 1, 1, None, base, 4, None) == -1                    # null in, n > 0
    assert L.sam_scan(1, 1, 1, 1, base + 4, base + 64, 4, None) == -1           # misaligned int64
    assert L.sam_scan(0, 1, 1, 1, base, base + 8, 16, None) == -1               # partial overlap
    assert L.sam_shard_scan(0, 1, 1, 1, base, base + 256, 4, 0, base, 3, 2, None) == -1  # rank >= nranks
    assert L.sam_scan(0, 1, 1, 1, None, None, 0, None) == 0                     # n == 0 is a no-op
    # delta encoder (not in place)
    assert L.sam_delta_encode(0, 1, 1, base, base, 4, None) == -1               # in place refused
    assert L.sam_delta_encode(0, 1, 1, base, base + 8, 16, None) == -1          # partial overlap
    assert L.sam_delta_encode(0, 9, 1, base, base + 256, 4, None) == -2         # order > 8
    assert L.sam_delta_encode(0, 1, 0, base, base + 256, 4, None) == -2         # tuple < 1
    assert L.sam_delta_encode(3, 1, 1, None, None, 0, None) == 0                # n == 0 is a no-op
    assert L.sam_delta_encode_host(0, 2, 2, base, base, 4, None) == -1          # host encoder: not in place
    assert L.sam_delta_encode_host(0, 0, 2, base, base + 256, 4, None) == -2    # order < 1
    assert L.sam_delta_encode_host(0, 1, 1, None, None, 0, None) == 0           # n == 0 is a no-op


@pytest.mark.parametrize("dt,k,s,expected", [(0, 1, 1, 32), (1, 4, 4, 144), (1, 8, 8, 528), (2, 3, 5, 80)])
def test_payload_bytes(dt, k, s, expected):
    S = _lib()
    assert S.sam_shard_payload_bytes(dt, k, s) == expected  # 16-B header + k*s values, 16-B aligned


def _payloads_from_oracle(x, bounds, k, s, name):
    """Shard payloads built with the ORACLE (test side): zero-seeded state of each global lane at
    its last element of the shard = the oracle's running sums after streaming the shard alone."""
    import paper_conf_pldi_malekiyb16_b200 as S

    dc = {"i32": 0, "i64": 1, "f32": 2, "f64": 3}[name]
    pb = S.sam_shard_payload_bytes(dc, k, s)
    w = np.dtype(x.dtype).itemsize
    buf = np.zeros((len(bounds) - 1) * pb, dtype=np.uint8)
    for r in range(len(bounds) - 1):
        lo, hi = bounds[r], bounds[r + 1]
        hdr = buf[r * pb: r * pb + 16].view(np.uint64)
        hdr[0], hdr[1] = hi - lo, lo
        _, run = oracle.scan(x[lo:hi], k, s, True, phase=lo % s)
        st = run.reshape(k, s).T.copy()  # [lane][order]
        if name == "f32":
            st = st.astype(np.float32)
        elif name == "f64":
            st = st.astype(np.float64)
        vals = buf[r * pb + 16: r * pb + 16 + k * s * w].view(x.dtype if name.startswith("i") else st.dtype)
        vals[:] = st.reshape(-1).view(vals.dtype) if name.startswith("i") else st.reshape(-1)
    return buf, pb, dc


@pytest.mark.parametrize("name", ["i32", "i64"])
@pytest.mark.parametrize("k,s", [(1, 1), (4, 4), (8, 8), (3, 5), (2, 7)])
def test_host_fold_matches_oracle_stream(name, k, s):
    """sam_fold_payloads_host (the carry operator M(L) S + P over shard payloads)
    reproduces the oracle's running state at each shard boundary, with uneven shards, empty
    shards and shard lengths not divisible by s (lanes absent from a shard pass through)."""
    S = _lib()
    n = 5003
    x = synth.make(n, name, "uniform", seed=k * 10 + s)
    bounds = [0, 1, 1, 17, 2500, 2501, 4000, n]
    buf, pb, dc = _payloads_from_oracle(x, bounds, k, s, name)
    ut = np.uint32 if name == "i32" else np.uint64
    for rank in range(len(bounds) - 1):
        seed = np.zeros(k * s, dtype=ut)
        S.sam_fold_payloads_host(dc, k, s, buf.ctypes.data, rank, len(bounds) - 1, seed.ctypes.data)
        _, run = oracle.scan(x[: bounds[rank]], k, s, True, phase=0)
        assert np.array_equal(seed.reshape(s, k), run.reshape(k, s).T), f"rank {rank}"


def test_host_fold_floats_close():
    S = _lib()
    k, s, n = 3, 2, 4001
    x = synth.make(n, "f64", "unif01", seed=3)
    bounds = [0, 1000, 1001, 3000, n]
    buf, pb, dc = _payloads_from_oracle(x, bounds, k, s, "f64")
    for rank in range(len(bounds) - 1):
        seed = np.zeros(k * s, dtype=np.float64)
        S.sam_fold_payloads_host(dc, k, s, buf.ctypes.data, rank, len(bounds) - 1, seed.ctypes.data)
        _, run = oracle.scan(x[: bounds[rank]], k, s, True, phase=0)
        ref = run.reshape(k, s).T.astype(np.float64)
        assert np.allclose(seed.reshape(s, k), ref, rtol=1e-12, atol=0)


def test_workspace_size_and_ws_validation():
    """sam_scan_workspace_size / sam_scan_ws: sizes grow with n and with k*s, and
    sam_scan_ws validates its workspace synchronously, before any CUDA call."""
    S = _lib()
    L = S.lib()
    sz = [S.sam_scan_workspace_size(S.SAM_I64, 4, 4, n) for n in (1, 1 << 20, 1 << 30, 1 << 33)]
    assert sz == sorted(sz) and sz[0] >= 1024
    assert S.sam_scan_workspace_size(S.SAM_I32, 8, 8, 1 << 20) >= S.sam_scan_workspace_size(S.SAM_I32, 1, 1, 1 << 20)
    with pytest.raises(S.SamError):
        S.sam_scan_workspace_size(S.SAM_I32, 9, 1, 10)
    buf = (ctypes.c_int64 * 512)()
    base = ctypes.addressof(buf)
    need = S.sam_scan_workspace_size(S.SAM_I32, 1, 1, 16)
    assert L.sam_scan_ws(0, 1, 1, 1, base, base + 2048, 16, None, need, None) == -1        # null ws
    assert L.sam_scan_ws(0, 1, 1, 1, base, base + 2048, 16, base + 8, need, None) == -1    # misaligned ws
    assert L.sam_scan_ws(0, 1, 1, 1, base, base + 2048, 16, base + 16, need - 8, None) == -1  # too small
    assert "workspace" in S.sam_last_error()
    assert L.sam_scan_ws(0, 1, 1, 1, base, base, 0, None, 0, None) == 0                   # n == 0: no-op
