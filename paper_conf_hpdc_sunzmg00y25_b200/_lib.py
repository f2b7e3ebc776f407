"""ctypes binding of libft2.so (include/ft2.h).  Argument marshalling only.

The library must have been built for sm_100a (``build.py``).  There is no
fallback: if the shared object is missing or fails to load, importing the
package raises.
"""
from __future__ import annotations

import ctypes
import os

from .build import LIB

FT2_OK, FT2_ERR_INVALID_ARG, FT2_ERR_MISALIGNED, FT2_ERR_UNSUPPORTED, FT2_ERR_CUDA = range(5)
FT2_BF16, FT2_FP16, FT2_FP32 = 0, 1, 2
FT2_FAULT_1BIT, FT2_FAULT_2BIT, FT2_FAULT_EXP = 0, 1, 2
FT2_GEMM_PLAIN, FT2_GEMM_CHECK, FT2_GEMM_W_STATIC = 0, 1, 16
FT2_MAX_SITE_LAYERS = 1024
FT2_MAX_SEQS = 65535


class Tensor(ctypes.Structure):
    _fields_ = [("data", ctypes.c_void_p), ("rows", ctypes.c_int64), ("n", ctypes.c_int64),
                ("ld", ctypes.c_int64), ("dtype", ctypes.c_int)]


class FaultSite(ctypes.Structure):
    _fields_ = [("trial", ctypes.c_uint32), ("step", ctypes.c_uint16), ("layer", ctypes.c_uint16),
                ("token", ctypes.c_uint32), ("col", ctypes.c_uint32), ("xor_mask", ctypes.c_uint32),
                ("model", ctypes.c_uint8), ("nbits", ctypes.c_uint8), ("pad", ctypes.c_uint8 * 2)]


class SiteGeometry(ctypes.Structure):
    _fields_ = [("n_steps", ctypes.c_int32), ("prompt_len", ctypes.c_int32), ("n_layers", ctypes.c_int32),
                ("layer_width", ctypes.POINTER(ctypes.c_int32)), ("layer_uniform", ctypes.c_int32),
                ("step_policy", ctypes.c_int32)]


assert ctypes.sizeof(FaultSite) == 24

EXPORTS = [
    "ft2_workspace_bytes", "ft2_bounds_from_prefill", "ft2_bounds_finalize", "ft2_protect",
    "ft2_gemm_workspace_bytes", "ft2_protect_fused_gemm", "ft2_protect_fused_gemm_ex", "ft2_prefill_fused_gemm", "ft2_make_fault_sites",
    "ft2_inject_faults", "ft2_allreduce_protect", "ft2_ipc_get_handle", "ft2_ipc_open_handle", "ft2_ipc_close",
    "ft2_status_string", "ft2_launch_count", "ft2_version", "ft2_host_norm", "ft2_host_act",
]

_lib = None


def load(path: str = LIB):
    """Load libft2.so and declare every entry point of include/ft2.h."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"libft2.so not built ({path}); run __graft_entry__.build()")
    L = ctypes.CDLL(path)
    P, i32, i64, u64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_float
    st = ctypes.c_int
    sig = {
        "ft2_workspace_bytes": (ctypes.c_size_t, [i32]),
        "ft2_bounds_from_prefill": (st, [Tensor, P, i32, f32, i32, i32, P, P, P, P, P, P]),
        "ft2_bounds_finalize": (st, [P, i32, f32, ctypes.c_int, P, P]),
        "ft2_protect": (st, [Tensor, P, P, i32, P, P]),
        "ft2_gemm_workspace_bytes": (ctypes.c_size_t, [i32, i32, i32]),
        "ft2_protect_fused_gemm": (st, [P, i64, P, i64, P, P, i64, i32, i32, i32, ctypes.c_int, ctypes.c_int, i32, i32,
                                        P, P, i32, P, P, i32, i32, i32, P, P, ctypes.c_size_t, P]),
        "ft2_protect_fused_gemm_ex": (st, [P, i64, P, i64, P, P, i64, i32, i32, i32, ctypes.c_int, ctypes.c_int, i32,
                                           i32, P, P, i32, P, P, i32, i32, i32, P, P, ctypes.c_size_t, P,
                                           ctypes.c_size_t, P]),
        "ft2_prefill_fused_gemm": (st, [P, i64, P, i64, P, P, i64, i32, i32, i32, ctypes.c_int, P, i32, f32, i32,
                                        P, P, P, P, i32, i32, P, P, P, ctypes.c_size_t, P]),
        "ft2_make_fault_sites": (st, [u64, u64, i32, ctypes.c_int, ctypes.c_int, ctypes.POINTER(SiteGeometry),
                                      P, P]),
        "ft2_inject_faults": (st, [Tensor, P, i32, i32, i32, P, P]),
        "ft2_allreduce_protect": (st, [P, i64, i32, i32, P, P, P, P, Tensor, P, ctypes.c_int, P, P, i32, P, P, i32,
                                       i32, i32, P, P]),
        "ft2_ipc_get_handle": (st, [P, P, ctypes.POINTER(ctypes.c_uint64)]),
        "ft2_ipc_open_handle": (st, [P, ctypes.POINTER(ctypes.c_void_p)]),
        "ft2_ipc_close": (st, [P]),
        "ft2_status_string": (ctypes.c_char_p, [ctypes.c_int]),
        "ft2_launch_count": (ctypes.c_uint64, []),
        "ft2_version": (ctypes.c_char_p, []),
        "ft2_host_norm": (st, [P, i64, P, P, P, i64, i64, i32, f32, ctypes.c_int, ctypes.c_int, P]),
        "ft2_host_act": (st, [P, i64, P, i64, P, i64, i64, i32, ctypes.c_int, ctypes.c_int, P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


class FT2Error(RuntimeError):
    def __init__(self, fn: str, status: int):
        msg = load().ft2_status_string(status).decode()
        super().__init__(f"{fn} -> {msg}")
        self.status = status


def check(fn: str, status: int):
    if status != FT2_OK:
        raise FT2Error(fn, status)
