"""FT2 CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package (``paper_conf_hpdc_sunzmg00y25_b200``) never imports it, and
``oracle/ft2_oracle.c`` shares no code with ``csrc/``.

Parity pins: every function here is pinned by ``tests/test_oracle_*.py``
against what the paper and the mathematics fix (Table 1, Fig. 7 closed forms,
the paper's CI margin, library routines ``torch.clamp``/``nan_to_num``/
``amin``/``amax``, ml_dtypes rounding, Philox known-answer vectors, brute
force).  Functions without such a pin say "parity unpinned" below:
  * campaign proxy-SDC rates / overhead % -- parity unpinned (need trained
    weights, datasets and the authors' hardware).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ft2_oracle.c")
_LIB = os.path.join(_HERE, "libft2_oracle.so")

SITE_DTYPE = np.dtype([
    ("trial", "<u4"), ("step", "<u2"), ("layer", "<u2"), ("token", "<u4"), ("col", "<u4"),
    ("xor_mask", "<u4"), ("model", "u1"), ("nbits", "u1"), ("pad", "u1", (2,)),
])
assert SITE_DTYPE.itemsize == 24

FAULT_1BIT, FAULT_2BIT, FAULT_EXP = 0, 1, 2
DT_BF16, DT_FP16, DT_FP32 = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C, IEEE fp, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fPIC", "-shared", "-fopenmp",
               "-fvisibility=hidden", "-std=c11", "-o", _LIB, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        u16, i32, i64, u32, u64 = (ctypes.c_uint16, ctypes.c_int32, ctypes.c_int64,
                                   ctypes.c_uint32, ctypes.c_uint64)
        P = ctypes.c_void_p
        for name, res, args in [
            ("ft2o_key", u16, [u16]), ("ft2o_unkey", u16, [u16]),
            ("ft2o_isnan", ctypes.c_int, [u16]), ("ft2o_isinf", ctypes.c_int, [u16]),
            ("ft2o_isfinite", ctypes.c_int, [u16]),
            ("ft2o_bf16_to_f64", ctypes.c_double, [u16]),
            ("ft2o_f64_to_bf16_rne", u16, [ctypes.c_double]),
            ("ft2o_f64_to_bf16_dir", u16, [ctypes.c_double, ctypes.c_int]),
            ("ft2o_scale_bound", u16, [u16, ctypes.c_float, ctypes.c_int]),
            ("ft2o_clip_value", u16, [u16, u16, u16]),
            ("ft2o_protect", None, [P, i64, i64, i64, P, P, i32, P]),
            ("ft2o_bounds", None, [P, i64, i64, i64, P, i32, ctypes.c_float, i32, P, P, P]),
            ("ft2o_bounds_from_keys", None, [P, i32, ctypes.c_float, P]),
            ("ft2o_philox4x32_10", None, [P, P, P]),
            ("ft2o_make_sites", None, [u64, u64, i32, i32, i32, i32, i32, i32, P, i32, i32, P]),
            ("ft2o_inject", None, [P, i64, i64, i64, P, i32, i32, i32, P]),
            ("ft2o_linear_f64", None, [P, i64, P, i64, P, i32, i32, i32, P, P, i64]),
            ("ft2o_protected_linear", None, [P, i64, P, i64, P, i32, i32, i32, P, i64, P, P, i32, P,
                                             P, i32, i32, i32, P]),
            ("ft2o_site_size", i32, []),
            ("ft2o_set_threads", None, [i32]), ("ft2o_max_threads", i32, []),
            ("ft2o_nan_vulnerable_count", None, [P, i64, i64, i64, P, i32, P, ctypes.c_int]),
            ("ft2o_isnan_dt", ctypes.c_int, [u16, ctypes.c_int]), ("ft2o_isinf_dt", ctypes.c_int, [u16, ctypes.c_int]),
            ("ft2o_isfinite_dt", ctypes.c_int, [u16, ctypes.c_int]),
            ("ft2o_to_f64_dt", ctypes.c_double, [u16, ctypes.c_int]),
            ("ft2o_f64_to_dt_rne", u16, [ctypes.c_double, ctypes.c_int]),
            ("ft2o_f64_to_dt_dir", u16, [ctypes.c_double, ctypes.c_int, ctypes.c_int]),
            ("ft2o_scale_bound_dt", u16, [u16, ctypes.c_float, ctypes.c_int, ctypes.c_int]),
            ("ft2o_clip_value_dt", u16, [u16, u16, u16, ctypes.c_int]),
            ("ft2o_protect_dt", None, [P, i64, i64, i64, P, P, i32, P, ctypes.c_int]),
            ("ft2o_bounds_dt", None, [P, i64, i64, i64, P, i32, ctypes.c_float, i32, P, P, P, ctypes.c_int]),
            ("ft2o_bounds_from_keys_dt", None, [P, i32, ctypes.c_float, P, ctypes.c_int]),
            ("ft2o_linear_f64_dt", None, [P, i64, P, i64, P, i32, i32, i32, P, P, i64, ctypes.c_int]),
            ("ft2o_protected_linear_dt", None, [P, i64, P, i64, P, i32, i32, i32, P, i64, P, P, i32, P,
                                                P, i32, i32, i32, P, ctypes.c_int]),
            ("ft2o_isnan32", ctypes.c_int, [u32]), ("ft2o_isfinite32", ctypes.c_int, [u32]),
            ("ft2o_key32", u32, [u32]), ("ft2o_unkey32", u32, [u32]),
            ("ft2o_scale_bound32", u32, [u32, ctypes.c_float, ctypes.c_int]),
            ("ft2o_clip_value32", u32, [u32, u32, u32]),
            ("ft2o_protect32", None, [P, i64, i64, i64, P, P, i32, P]),
            ("ft2o_bounds32", None, [P, i64, i64, i64, P, i32, ctypes.c_float, i32, P, P, P, P]),
            ("ft2o_inject32", None, [P, i64, i64, i64, P, i32, i32, i32, P]),
            ("ft2o_allreduce_protect", None, [P, i32, i64, i64, P, i32, P, P, i32, P, P, i32, i32, i32, P, P,
                                              ctypes.c_int]),
        ]:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        assert L.ft2o_site_size() == SITE_DTYPE.itemsize
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _u16(a):
    a = np.ascontiguousarray(a)
    if a.dtype != np.uint16:
        a = a.view(np.uint16) if a.dtype.itemsize == 2 else a.astype(np.uint16)
    return a


# ----------------------------------------------------------------- scalars --
def isnan_dt(b: int, dtype: int) -> bool: return bool(lib().ft2o_isnan_dt(b, dtype))
def isinf_dt(b: int, dtype: int) -> bool: return bool(lib().ft2o_isinf_dt(b, dtype))
def to_f64(b: int, dtype: int = DT_BF16) -> float: return lib().ft2o_to_f64_dt(b, dtype)
def f64_to(d: float, dtype: int = DT_BF16) -> int: return lib().ft2o_f64_to_dt_rne(d, dtype)
def f64_to_dir(d: float, direction: int, dtype: int = DT_BF16) -> int: return lib().ft2o_f64_to_dt_dir(d, direction, dtype)
def key(b: int) -> int: return lib().ft2o_key(b)
def unkey(k: int) -> int: return lib().ft2o_unkey(k)
def isnan(b: int) -> bool: return bool(lib().ft2o_isnan(b))
def isinf(b: int) -> bool: return bool(lib().ft2o_isinf(b))
def bf16_to_f64(b: int) -> float: return lib().ft2o_bf16_to_f64(b)
def f64_to_bf16(d: float) -> int: return lib().ft2o_f64_to_bf16_rne(d)
def f64_to_bf16_dir(d: float, direction: int) -> int: return lib().ft2o_f64_to_bf16_dir(d, direction)
def scale_bound(raw: int, c: float, is_hi: bool, dtype: int = DT_BF16) -> int:
    return lib().ft2o_scale_bound_dt(raw, c, int(is_hi), dtype)
def clip_value(y: int, lo: int, hi: int, dtype: int = DT_BF16) -> int: return lib().ft2o_clip_value_dt(y, lo, hi, dtype)


def philox4x32_10(ctr, key_):
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key_, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().ft2o_philox4x32_10(_p(c), _p(k), _p(out))
    return [int(x) for x in out]


# ------------------------------------------------------------------ tensors --
def bounds(y, seq_offsets=None, scale: float = 2.0, correct_nonfinite: bool = False, ld=None, dtype=DT_BF16):
    """R2-R4.  y: uint16 [rows, n] (modified in place iff correct_nonfinite).

    Returns (bounds uint16 [S,2], raw_keys int32 [S,2], nonfinite uint32 [S]).
    """
    assert y.dtype == np.uint16 and y.ndim == 2 and y.flags.c_contiguous
    rows, n = y.shape
    ld = n if ld is None else ld
    so = None if seq_offsets is None else np.ascontiguousarray(seq_offsets, dtype=np.int32)
    S = 1 if so is None else so.size - 1
    b = np.zeros((S, 2), np.uint16)
    k = np.zeros((S, 2), np.int32)
    nf = np.zeros(S, np.uint32)
    lib().ft2o_bounds_dt(_p(y), rows, n, ld, _p(so), S, scale, int(correct_nonfinite), _p(b), _p(k), _p(nf), dtype)
    return b, k, nf


def nan_vulnerable_count(y, seq_offsets=None, dtype=DT_BF16):
    """Per-sequence count of values in (-2,-1) U (1,2)."""
    y = np.ascontiguousarray(y, dtype=np.uint16)
    so = None if seq_offsets is None else np.ascontiguousarray(seq_offsets, dtype=np.int32)
    S = 1 if so is None else so.size - 1
    out = np.zeros(S, np.uint32)
    lib().ft2o_nan_vulnerable_count(_p(y), y.shape[0], y.shape[1], y.shape[1], _p(so), S, _p(out), dtype)
    return out


def bounds_from_keys(raw_keys, scale: float = 2.0, dtype=DT_BF16):
    k = np.ascontiguousarray(raw_keys, dtype=np.int32)
    S = k.shape[0]
    b = np.zeros((S, 2), np.uint16)
    lib().ft2o_bounds_from_keys_dt(_p(k), S, scale, _p(b), dtype)
    return b


def set_threads(n: int) -> int:
    """OpenMP threads for the oracle's loops over independent outputs (results
    are identical for any count); n < 1 = all cores.  Returns the count now in use."""
    lib().ft2o_set_threads(int(n))
    return int(lib().ft2o_max_threads())


def protect(y, bounds_, row_to_seq=None, count=None, dtype=DT_BF16):
    """R5 in place.  y: uint16 [rows, n]; bounds_: uint16 [S, 2]. Returns count [S]."""
    assert y.dtype == np.uint16 and y.ndim == 2 and y.flags.c_contiguous
    rows, n = y.shape
    b = np.ascontiguousarray(bounds_, dtype=np.uint16)
    S = b.shape[0]
    r2s = None if row_to_seq is None else np.ascontiguousarray(row_to_seq, dtype=np.int32)
    if count is None:
        count = np.zeros(S, np.uint32)
    lib().ft2o_protect_dt(_p(y), rows, n, n, _p(r2s), _p(b), S, _p(count), dtype)
    return count


def make_sites(seed, trial0, n_trials, model, layer_width, n_steps, prompt_len,
               dtype=DT_BF16, layer_uniform=True, step_policy=0):
    w = np.ascontiguousarray(layer_width, dtype=np.int32)
    out = np.zeros(n_trials, SITE_DTYPE)
    lib().ft2o_make_sites(seed, trial0, n_trials, model, dtype, n_steps, prompt_len, w.size,
                          _p(w), int(layer_uniform), int(step_policy), _p(out))
    return out


def inject(y, sites, cur_layer, cur_step, base_row=None):
    assert y.dtype == np.uint16 and y.ndim == 2 and y.flags.c_contiguous
    s = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    br = None if base_row is None else np.ascontiguousarray(base_row, dtype=np.int32)
    lib().ft2o_inject(_p(y), y.shape[0], y.shape[1], y.shape[1], _p(s), s.size, cur_layer, cur_step, _p(br))
    return y


def linear_f64(x, w, bias=None, dtype=DT_BF16):
    """R8: returns (y_f64 [M,N], y rounded to the activation dtype [M,N] as uint16 bits)."""
    x = _u16(x)
    w = _u16(w)
    M, K = x.shape
    N = w.shape[0]
    b = None if bias is None else _u16(bias)
    yd = np.zeros((M, N), np.float64)
    yb = np.zeros((M, N), np.uint16)
    lib().ft2o_linear_f64_dt(_p(x), K, _p(w), K, _p(b), M, N, K, _p(yd), _p(yb), N, dtype)
    return yd, yb


def protected_linear(x, w, bias, bounds_, row_to_seq=None, sites=None, cur_layer=0, cur_step=0,
                     base_row=None, dtype=DT_BF16):
    """R8 -> R7 -> R5. Returns (y bf16 [M,N], count [S])."""
    x = _u16(x)
    w = _u16(w)
    M, K = x.shape
    N = w.shape[0]
    b = None if bias is None else _u16(bias)
    bd = np.ascontiguousarray(bounds_, dtype=np.uint16)
    S = bd.shape[0]
    y = np.zeros((M, N), np.uint16)
    cnt = np.zeros(S, np.uint32)
    r2s = None if row_to_seq is None else np.ascontiguousarray(row_to_seq, dtype=np.int32)
    s = None if sites is None else np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    ns = 0 if s is None else s.size
    br = None if base_row is None else np.ascontiguousarray(base_row, dtype=np.int32)
    lib().ft2o_protected_linear_dt(_p(x), K, _p(w), K, _p(b), M, N, K, _p(y), N, _p(r2s), _p(bd), S,
                                   _p(cnt), _p(s), ns, cur_layer, cur_step, _p(br), dtype)
    return y, cnt


# ------------------------------------------------------------------- FP32 --
# The paper's FP32 study: the same method on binary32
# activations, handled as uint32 bit patterns with a 32-bit order key.
def key32(b: int) -> int: return lib().ft2o_key32(b)
def unkey32(k: int) -> int: return lib().ft2o_unkey32(k)
def isnan32(b: int) -> bool: return bool(lib().ft2o_isnan32(b))
def scale_bound32(raw: int, c: float, is_hi: bool) -> int: return lib().ft2o_scale_bound32(raw, c, int(is_hi))
def clip_value32(y: int, lo: int, hi: int) -> int: return lib().ft2o_clip_value32(y, lo, hi)


def _u32(a):
    a = np.ascontiguousarray(a)
    if a.dtype != np.uint32:
        a = a.view(np.uint32) if a.dtype.itemsize == 4 else a.astype(np.uint32)
    return a


def bounds32(y, seq_offsets=None, scale: float = 2.0, correct_nonfinite: bool = False):
    """R2-R4 on binary32 bits y (uint32 [rows, n], modified in place iff
    correct_nonfinite).  Returns (bounds uint32 [S,2], raw keys uint32 [S,2],
    have int32 [S], nonfinite uint32 [S])."""
    assert y.dtype == np.uint32 and y.ndim == 2 and y.flags.c_contiguous
    rows, n = y.shape
    so = None if seq_offsets is None else np.ascontiguousarray(seq_offsets, dtype=np.int32)
    S = 1 if so is None else so.size - 1
    b = np.zeros((S, 2), np.uint32)
    k = np.zeros((S, 2), np.uint32)
    have = np.zeros(S, np.int32)
    nf = np.zeros(S, np.uint32)
    lib().ft2o_bounds32(_p(y), rows, n, n, _p(so), S, scale, int(correct_nonfinite), _p(b), _p(k), _p(have), _p(nf))
    return b, k, have, nf


def protect32(y, bounds_, row_to_seq=None, count=None):
    """R5 in place on binary32 bits y (uint32 [rows, n]); bounds_ uint32 [S, 2]."""
    assert y.dtype == np.uint32 and y.ndim == 2 and y.flags.c_contiguous
    rows, n = y.shape
    b = _u32(bounds_).reshape(-1, 2)
    S = b.shape[0]
    cnt = np.zeros(S, np.uint32) if count is None else count
    r2s = None if row_to_seq is None else np.ascontiguousarray(row_to_seq, dtype=np.int32)
    lib().ft2o_protect32(_p(y), rows, n, n, _p(r2s), _p(b), S, _p(cnt))
    return cnt


def inject32(y, sites, cur_layer, cur_step, base_row=None):
    assert y.dtype == np.uint32 and y.ndim == 2 and y.flags.c_contiguous
    rows, n = y.shape
    s = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    br = None if base_row is None else np.ascontiguousarray(base_row, dtype=np.int32)
    lib().ft2o_inject32(_p(y), rows, n, n, _p(s), s.size, cur_layer, cur_step, _p(br))
    return y


def allreduce_protect(partials, bias=None, bounds_=None, row_to_seq=None, sites=None, cur_layer=0, cur_step=0,
                      base_row=None, dtype=DT_BF16):
    """Reading A22 + A17: partials uint16 [P, rows, n] -> (y uint16 [rows, n], count [S])."""
    pp = np.ascontiguousarray(partials, dtype=np.uint16)
    P, rows, n = pp.shape
    y = np.zeros((rows, n), np.uint16)
    b = None if bias is None else np.ascontiguousarray(bias, dtype=np.uint16)
    bd = None if bounds_ is None else np.ascontiguousarray(bounds_, dtype=np.uint16).reshape(-1, 2)
    S = 0 if bd is None else bd.shape[0]
    cnt = np.zeros(max(S, 1), np.uint32)
    r2s = None if row_to_seq is None else np.ascontiguousarray(row_to_seq, dtype=np.int32)
    s = None if sites is None else np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    br = None if base_row is None else np.ascontiguousarray(base_row, dtype=np.int32)
    lib().ft2o_allreduce_protect(_p(pp), P, rows, n, _p(b), int(bd is not None), _p(r2s), _p(bd), S, _p(cnt),
                                 _p(s), 0 if s is None else s.size, cur_layer, cur_step, _p(br), _p(y), dtype)
    return y, cnt[:S]
