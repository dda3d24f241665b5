"""sam-b200: single-pass higher-order / tuple-based prefix sums on B200 (sm_100a).

Thin Python binding over the C ABI of libsam.so (include/sam.h).  The functions named like the
C entry points (sam_scan, sam_scan_seeded, sam_shard_state, ...) marshal arguments only; every
step of the scan runs in the library's CUDA kernels.  torch is used for device memory, streams
and (dist.py) process groups.  There is no CPU fallback: if libsam.so is missing or no CUDA
device is present, calls raise.

Method: Maleki, Yang & Burtscher, PLDI'16; semantics in include/sam.h and DESIGN.md.
"""
from __future__ import annotations

import ctypes
import os

__all__ = [
    "SamError", "lib", "SAM_I32", "SAM_I64", "SAM_F32", "SAM_F64",
    "sam_scan", "sam_scan_seeded", "sam_scan_host", "sam_prepare", "sam_scan_workspace_size", "sam_scan_ws",
    "sam_debug_limit_grid", "sam_debug_set_stress", "sam_scan_op", "sam_scan_generic", "sam_last_carry_scheme", "sam_tune_override", "sam_debug_last_shape",
    "scan_op", "SAM_U32", "SAM_U64", "SAM_OP", "SAM_CARRY", "sam_shard_payload_bytes",
    "sam_shard_state", "sam_shard_scan", "sam_fold_payloads_host", "sam_last_error", "sam_version",
    "sam_launch_count", "sam_release_workspaces", "sam_delta_encode", "sam_delta_encode_halo", "sam_delta_encode_host", "delta_encode_host", "scan", "delta_encode", "scan_host", "dtype_code", "LIB_PATH",
]

SAM_I32, SAM_I64, SAM_F32, SAM_F64, SAM_U32, SAM_U64 = 0, 1, 2, 3, 4, 5
SAM_OP = {"add": 0, "xor": 1, "max": 2, "min": 3}
SAM_CARRY = {"static": 0, "lookback": 1, "chained": 2}
_STATUS = {0: "SAM_OK", -1: "SAM_ERR_INVALID_ARG", -2: "SAM_ERR_UNSUPPORTED", -3: "SAM_ERR_CUDA",
           -4: "SAM_ERR_OOM", -5: "SAM_ERR_INTERNAL"}

LIB_PATH = os.environ.get("SAM_LIB_PATH") or \
    os.path.join(os.path.dirname(os.path.abspath(__file__)), "lib", "libsam.so")  # override: experiments
_lib = None


class SamError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_STATUS.get(code, code)}: {msg}")
        self.code = code


def lib() -> ctypes.CDLL:
    """Load libsam.so (fails loudly if it has not been built: python -m paper_conf_pldi_malekiyb16_b200._build)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libsam.so not found at {LIB_PATH}; build it with "
                               "`python -m paper_conf_pldi_malekiyb16_b200._build` (or __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        P, I, U64, SZ = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64, ctypes.c_size_t
        sig = {
            "sam_scan": (I, [I, I, I, I, P, P, U64, P]),
            "sam_scan_seeded": (I, [I, I, I, I, P, P, U64, U64, P, P, P]),
            "sam_prepare": (I, [I, I, I, U64, P]),
            "sam_scan_host": (I, [I, I, I, I, P, P, U64, P]),
            "sam_shard_payload_bytes": (SZ, [I, I, I]),
            "sam_shard_state": (I, [I, I, I, P, U64, U64, P, P]),
            "sam_shard_scan": (I, [I, I, I, I, P, P, U64, U64, P, I, I, P]),
            "sam_fold_payloads_host": (I, [I, I, I, P, I, I, P]),
            "sam_cyclic_fold": (I, [I, I, I, P, I, I, P, P, P, P]),
            "sam_cyclic_fold_host": (I, [I, I, I, P, I, I, P, P, P]),
            "sam_delta_encode": (I, [I, I, I, P, P, U64, P]),
            "sam_delta_encode_halo": (I, [I, I, I, P, P, U64, P, P]),
            "sam_delta_encode_host": (I, [I, I, I, P, P, U64, P]),
            "sam_last_error": (ctypes.c_char_p, []),
            "sam_version": (ctypes.c_char_p, []),
            "sam_release_workspaces": (I, []),
            "sam_launch_count": (U64, []),
            "sam_debug_set_trace": (I, [P]),
            "sam_debug_limit_grid": (I, [U64]),
            "sam_scan_op": (I, [I, I, I, I, I, P, P, U64, P]),
            "sam_scan_generic": (I, [I, I, I, I, I, I, P, P, U64, P]),
            "sam_last_carry_scheme": (I, []),
            "sam_tune_override": (I, [I, I, I, I, I]),
            "sam_debug_last_shape": (I, [ctypes.POINTER(ctypes.c_int)]),
            "sam_debug_set_stress": (I, [ctypes.c_uint32]),
            "sam_scan_workspace_size": (I, [I, I, I, U64, ctypes.POINTER(SZ)]),
            "sam_scan_ws": (I, [I, I, I, I, P, P, U64, P, SZ, P]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name, None)
            if fn is None:  # an older library build (experiments via SAM_LIB_PATH)
                continue
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _check(rc: int) -> int:
    if rc != 0:
        raise SamError(rc, lib().sam_last_error().decode())
    return rc


# ----------------------------------------------------------------------------- raw C-ABI names
def sam_scan(dtype, order, tuple_, inclusive, in_ptr, out_ptr, n, stream=None) -> int:
    return _check(lib().sam_scan(dtype, order, tuple_, int(bool(inclusive)), in_ptr, out_ptr, n, stream))


def sam_scan_seeded(dtype, order, tuple_, inclusive, in_ptr, out_ptr, n, global_offset, seed_ptr,
                    final_ptr, stream=None) -> int:
    return _check(lib().sam_scan_seeded(dtype, order, tuple_, int(bool(inclusive)), in_ptr, out_ptr, n,
                                        global_offset, seed_ptr, final_ptr, stream))


def sam_scan_host(dtype, order, tuple_, inclusive, in_host_ptr, out_host_ptr, n, stream=None) -> int:
    return _check(lib().sam_scan_host(dtype, order, tuple_, int(bool(inclusive)), in_host_ptr, out_host_ptr, n,
                                      stream))


def sam_scan_workspace_size(dtype, order, tuple_, n) -> int:
    b = ctypes.c_size_t(0)
    _check(lib().sam_scan_workspace_size(dtype, order, tuple_, n, ctypes.byref(b)))
    return int(b.value)


def sam_scan_ws(dtype, order, tuple_, inclusive, in_ptr, out_ptr, n, ws_ptr, ws_bytes, stream=None) -> int:
    return _check(lib().sam_scan_ws(dtype, order, tuple_, int(bool(inclusive)), in_ptr, out_ptr, n, ws_ptr,
                                    ws_bytes, stream))


def sam_scan_op(dtype, op, order, tuple_, inclusive, in_ptr, out_ptr, n, stream=None) -> int:
    return _check(lib().sam_scan_op(dtype, op, order, tuple_, int(bool(inclusive)), in_ptr, out_ptr, n, stream))


def sam_scan_generic(dtype, op, carry, order, tuple_, inclusive, in_ptr, out_ptr, n, stream=None) -> int:
    return _check(lib().sam_scan_generic(dtype, op, carry, order, tuple_, int(bool(inclusive)), in_ptr, out_ptr, n,
                                         stream))


def sam_tune_override(tiles_per_unit=-1, lag=-1, vfold=-1, land=-1, teams=-1) -> int:
    return _check(lib().sam_tune_override(tiles_per_unit, lag, vfold, land, teams))


def sam_debug_last_shape() -> dict:
    v = (ctypes.c_int * 6)()
    _check(lib().sam_debug_last_shape(v))
    return dict(zip(("M", "lag", "vfold", "land", "grid", "items"), list(v)))


def sam_last_carry_scheme() -> int:
    return int(lib().sam_last_carry_scheme())


def sam_debug_limit_grid(max_ctas: int) -> int:
    return _check(lib().sam_debug_limit_grid(max_ctas))


def sam_debug_set_stress(seed: int) -> int:
    return _check(lib().sam_debug_set_stress(seed))


def sam_prepare(dtype, order, tuple_, max_n, stream=None) -> int:
    return _check(lib().sam_prepare(dtype, order, tuple_, max_n, stream))


def sam_shard_payload_bytes(dtype, order, tuple_) -> int:
    return int(lib().sam_shard_payload_bytes(dtype, order, tuple_))


def sam_shard_state(dtype, order, tuple_, in_ptr, n_local, global_offset, payload_ptr, stream=None) -> int:
    return _check(lib().sam_shard_state(dtype, order, tuple_, in_ptr, n_local, global_offset, payload_ptr, stream))


def sam_shard_scan(dtype, order, tuple_, inclusive, in_ptr, out_ptr, n_local, global_offset, payloads_ptr,
                   rank, nranks, stream=None) -> int:
    return _check(lib().sam_shard_scan(dtype, order, tuple_, int(bool(inclusive)), in_ptr, out_ptr, n_local,
                                       global_offset, payloads_ptr, rank, nranks, stream))


def sam_fold_payloads_host(dtype, order, tuple_, payloads_host_ptr, rank, nranks, seed_host_ptr) -> int:
    return _check(lib().sam_fold_payloads_host(dtype, order, tuple_, payloads_host_ptr, rank, nranks, seed_host_ptr))


def sam_cyclic_fold(dtype, order, tuple_, round_payloads_ptr, rank, nranks, base_in_ptr, seed_out_ptr,
                    base_out_ptr, stream=None) -> int:
    return _check(lib().sam_cyclic_fold(dtype, order, tuple_, round_payloads_ptr, rank, nranks, base_in_ptr,
                                        seed_out_ptr, base_out_ptr, stream))


def sam_cyclic_fold_host(dtype, order, tuple_, round_payloads_host_ptr, rank, nranks, base_in_host_ptr,
                         seed_out_host_ptr, base_out_host_ptr) -> int:
    return _check(lib().sam_cyclic_fold_host(dtype, order, tuple_, round_payloads_host_ptr, rank, nranks,
                                             base_in_host_ptr, seed_out_host_ptr, base_out_host_ptr))


def sam_delta_encode(dtype, order, tuple_, in_ptr, out_ptr, n, stream=None) -> int:
    return _check(lib().sam_delta_encode(dtype, order, tuple_, in_ptr, out_ptr, n, stream))


def sam_delta_encode_halo(dtype, order, tuple_, in_ptr, out_ptr, n, halo_ptr, stream=None) -> int:
    return _check(lib().sam_delta_encode_halo(dtype, order, tuple_, in_ptr, out_ptr, n, halo_ptr, stream))


def sam_delta_encode_host(dtype, order, tuple_, in_host_ptr, out_host_ptr, n, stream=None) -> int:
    return _check(lib().sam_delta_encode_host(dtype, order, tuple_, in_host_ptr, out_host_ptr, n, stream))


def sam_last_error() -> str:
    return lib().sam_last_error().decode()


def sam_version() -> str:
    return lib().sam_version().decode()


def sam_launch_count() -> int:
    return int(lib().sam_launch_count())


def sam_release_workspaces() -> int:
    return _check(lib().sam_release_workspaces())


# ----------------------------------------------------------------------------- torch helpers
def dtype_code(dt) -> int:
    import torch

    m = {torch.int32: SAM_I32, torch.int64: SAM_I64, torch.float32: SAM_F32, torch.float64: SAM_F64}
    for name, code in (("uint32", SAM_U32), ("uint64", SAM_U64)):
        if hasattr(torch, name):
            m[getattr(torch, name)] = code
    if dt not in m:
        raise SamError(-2, f"unsupported dtype {dt} (int32, int64, float32, float64)")
    return m[dt]


def _stream_ptr(stream=None):
    import torch

    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def scan(x, order: int = 1, tuple: int = 1, inclusive: bool = True, out=None, stream=None):
    """Order-`order`, tuple-`tuple` prefix sum of a 1-D contiguous CUDA tensor (P:115-133,
    P:349-355).  `out` may be `x` (in place).  Asynchronous on the current stream."""
    if not x.is_cuda:
        raise SamError(-1, "scan() needs a CUDA tensor (use scan_host for host buffers)")
    if x.dim() != 1 or not x.is_contiguous():
        raise SamError(-1, "x must be 1-D and contiguous")
    if out is None:
        import torch

        out = torch.empty_like(x)
    sam_scan(dtype_code(x.dtype), order, tuple, inclusive, ctypes.c_void_p(x.data_ptr()),
             ctypes.c_void_p(out.data_ptr()), x.numel(), _stream_ptr(stream))
    return out


def scan_op(x, op: str = "add", order: int = 1, tuple: int = 1, inclusive: bool = True, out=None, stream=None,
            carry: str | None = None):
    """Order-`order`, tuple-`tuple` scan of a 1-D contiguous CUDA tensor under `op` in
    {"add", "xor", "max", "min"} (sam_scan_op).  `carry` in {"static", "lookback",
    "chained"} selects the generic kernel's carry scheme explicitly (sam_scan_generic, the NEXT-3
    ablation); None = the library's default path for the operator."""
    if not x.is_cuda or x.dim() != 1 or not x.is_contiguous():
        raise SamError(-1, "scan_op() needs a 1-D contiguous CUDA tensor")
    if op not in SAM_OP:
        raise SamError(-2, f"unknown operator {op!r}")
    if out is None:
        import torch

        out = torch.empty_like(x)
    args = (order, tuple, inclusive, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(out.data_ptr()), x.numel(),
            _stream_ptr(stream))
    if carry is None:
        sam_scan_op(dtype_code(x.dtype), SAM_OP[op], *args)
    else:
        if carry not in SAM_CARRY:
            raise SamError(-2, f"unknown carry scheme {carry!r}")
        sam_scan_generic(dtype_code(x.dtype), SAM_OP[op], SAM_CARRY[carry], *args)
    return out


def delta_encode(x, order: int = 1, tuple: int = 1, out=None, stream=None, halo=None):
    """Order-`order`, tuple-`tuple` difference sequence of a 1-D contiguous CUDA tensor
    (sam_delta_encode): the inverse of scan(..., inclusive=True).  Not in place.
    `halo`: optional CUDA tensor of the order*tuple elements preceding x (sam_delta_encode_halo)."""
    if not x.is_cuda or x.dim() != 1 or not x.is_contiguous():
        raise SamError(-1, "delta_encode() needs a 1-D contiguous CUDA tensor")
    if out is None:
        import torch

        out = torch.empty_like(x)
    if halo is not None:
        if not halo.is_cuda or halo.dtype != x.dtype or halo.numel() != order * tuple or not halo.is_contiguous():
            raise SamError(-1, "halo must be a contiguous CUDA tensor of order*tuple elements of x's dtype")
        hp = ctypes.c_void_p(halo.data_ptr())
    else:
        hp = None
    sam_delta_encode_halo(dtype_code(x.dtype), order, tuple, ctypes.c_void_p(x.data_ptr()),
                          ctypes.c_void_p(out.data_ptr()), x.numel(), hp, _stream_ptr(stream))
    return out


def delta_encode_host(x, order: int = 1, tuple: int = 1, out=None, stream=None):
    """End-to-end delta encoding of a host (CPU) tensor through the GPU (sam_delta_encode_host:
    chunked H2D | encode | D2H pipeline).  Pinned memory gives full PCIe bandwidth.  Synchronous."""
    import torch

    if x.is_cuda or x.dim() != 1 or not x.is_contiguous():
        raise SamError(-1, "delta_encode_host() needs a 1-D contiguous CPU tensor")
    if out is None:
        out = torch.empty_like(x)
    sam_delta_encode_host(dtype_code(x.dtype), order, tuple, ctypes.c_void_p(x.data_ptr()),
                          ctypes.c_void_p(out.data_ptr()), x.numel(), _stream_ptr(stream))
    return out


def scan_host(x, order: int = 1, tuple: int = 1, inclusive: bool = True, out=None, stream=None):
    """End-to-end scan of a host (CPU) tensor through the GPU: chunked H2D | scan | D2H pipeline
    (sam_scan_host).  Pinned memory gives full PCIe bandwidth.  Synchronous."""
    import torch

    if x.is_cuda or x.dim() != 1 or not x.is_contiguous():
        raise SamError(-1, "scan_host() needs a 1-D contiguous CPU tensor")
    if out is None:
        out = torch.empty_like(x)
    sam_scan_host(dtype_code(x.dtype), order, tuple, inclusive, ctypes.c_void_p(x.data_ptr()),
                  ctypes.c_void_p(out.data_ptr()), x.numel(), _stream_ptr(stream))
    return out


def tile_items(dtype_name: str) -> int:
    """Items per thread of the kernel's tile geometry (mirrors sam::Cfg<T>::ITEMS; tests use it to
    place sizes at tile boundaries)."""
    return {"i32": 27, "f32": 27, "i64": 13, "f64": 13}[dtype_name]
