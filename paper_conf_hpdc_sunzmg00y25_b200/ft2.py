"""torch-facing binding of libft2.so: same names as include/ft2.h, arguments
marshalled from torch tensors (data_ptr, shape, stride) and the current CUDA
stream.  No computation happens here -- every step runs in the library's
kernels.  PAPER.md citations are in include/ft2.h.
"""
from __future__ import annotations

import ctypes

import torch

from . import _lib
from ._lib import (FT2_BF16, FT2_FP16, FT2_FP32, FT2_GEMM_CHECK, FT2_GEMM_PLAIN, FaultSite, SiteGeometry, Tensor, check,
                   load)

_DTYPES = {torch.bfloat16: FT2_BF16, torch.float16: FT2_FP16, torch.float32: FT2_FP32}


def _dtype_of(t: torch.Tensor) -> int:
    if t.dtype not in _DTYPES:
        raise TypeError(f"ft2: unsupported activation dtype {t.dtype} (bfloat16 / float16 / float32)")
    return _DTYPES[t.dtype]

SITE_BYTES = ctypes.sizeof(FaultSite)


def _stream(stream=None):
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _as_ft2_tensor(y: torch.Tensor) -> Tensor:
    dt = _dtype_of(y)
    if not y.is_cuda:
        raise ValueError("ft2: tensor must live on a CUDA device (no CPU fallback)")
    if y.dim() == 1:
        y = y.view(1, -1)
    if y.dim() != 2:
        y2 = y.reshape(-1, y.shape[-1])
        if y2.data_ptr() != y.data_ptr():
            raise ValueError("ft2: tensor must be viewable as 2-D without a copy")
        y = y2
    if y.stride(1) != 1:
        raise ValueError("ft2: rows must be contiguous (stride(-1) == 1)")
    return Tensor(y.data_ptr(), y.shape[0], y.shape[1], y.stride(0), dt)


def workspace_bytes(num_seqs: int) -> int:
    return int(load().ft2_workspace_bytes(num_seqs))


def make_workspace(num_seqs: int, device=None) -> torch.Tensor:
    """Zero-filled workspace for ft2_bounds_from_prefill (self-cleaning afterwards)."""
    n = workspace_bytes(num_seqs)
    return torch.zeros((n + 7) // 8, dtype=torch.int64, device=device or "cuda")


def bounds_from_prefill(y, bounds_out, workspace, seq_offsets=None, num_seqs=None, scale=2.0,
                        finalize=True, correct_nonfinite=False, keys_out=None, nonfinite_count=None,
                        nan_vulnerable_count=None, stream=None):
    """ft2_bounds_from_prefill.  bounds_out: bf16 [S, 2] (or None when finalize=False)."""
    t = _as_ft2_tensor(y)
    S = num_seqs if num_seqs is not None else (1 if seq_offsets is None else seq_offsets.numel() - 1)
    st = load().ft2_bounds_from_prefill(t, _ptr(seq_offsets), S, float(scale), int(finalize),
                                        int(correct_nonfinite), _ptr(bounds_out), _ptr(keys_out),
                                        _ptr(nonfinite_count), _ptr(nan_vulnerable_count), _ptr(workspace),
                                        _stream(stream))
    check("ft2_bounds_from_prefill", st)


def bounds_finalize(keys, bounds_out, scale=2.0, stream=None):
    S = keys.numel() // 2
    check("ft2_bounds_finalize", load().ft2_bounds_finalize(_ptr(keys), S, float(scale), _dtype_of(bounds_out),
                                                            _ptr(bounds_out), _stream(stream)))


def protect(y, bounds, row_to_seq=None, num_seqs=None, corrected_count=None, stream=None):
    """ft2_protect, in place on y (bf16 [rows, n])."""
    t = _as_ft2_tensor(y)
    S = num_seqs if num_seqs is not None else bounds.numel() // 2
    check("ft2_protect", load().ft2_protect(t, _ptr(row_to_seq), _ptr(bounds), S, _ptr(corrected_count),
                                            _stream(stream)))


def protect_fused_gemm(x, w, y, bias=None, mode=FT2_GEMM_CHECK, bounds=None, row_to_seq=None, num_seqs=None,
                       corrected_count=None, col_begin=0, col_end=None, sites=None, n_sites=None,
                       cur_layer=0, cur_step=0, base_row=None, workspace=None, l2_prefetch=None, stream=None):
    """ft2_protect_fused_gemm: y = check(inject(bf16(x @ w.T + bias))).
    l2_prefetch: optional tensor (e.g. the next layer's weights) passed to
    ft2_protect_fused_gemm_ex as an L2 prefetch hint (its whole storage)."""
    M, K = x.shape
    N = w.shape[0]
    if col_end is None:
        col_end = N
    S = num_seqs if num_seqs is not None else (bounds.numel() // 2 if bounds is not None else 0)
    ns = 0 if sites is None else (n_sites if n_sites is not None else sites.numel() // SITE_BYTES)
    if workspace is None:
        workspace = default_gemm_workspace(x.device)
    ws = workspace.numel() * workspace.element_size()
    if l2_prefetch is None:
        st = load().ft2_protect_fused_gemm(_ptr(x), x.stride(0), _ptr(w), w.stride(0), _ptr(bias), _ptr(y),
                                           y.stride(0), M, N, K, int(mode), _dtype_of(x), col_begin, col_end,
                                           _ptr(row_to_seq), _ptr(bounds), S, _ptr(corrected_count), _ptr(sites), ns,
                                           cur_layer, cur_step, _ptr(base_row), _ptr(workspace), ws, _stream(stream))
        check("ft2_protect_fused_gemm", st)
        return
    assert l2_prefetch.is_contiguous(), "l2_prefetch must be a contiguous tensor"
    pf_bytes = (l2_prefetch.numel() * l2_prefetch.element_size()) & ~15
    st = load().ft2_protect_fused_gemm_ex(_ptr(x), x.stride(0), _ptr(w), w.stride(0), _ptr(bias), _ptr(y),
                                          y.stride(0), M, N, K, int(mode), _dtype_of(x), col_begin, col_end,
                                          _ptr(row_to_seq), _ptr(bounds), S, _ptr(corrected_count), _ptr(sites), ns,
                                          cur_layer, cur_step, _ptr(base_row), _ptr(workspace), ws,
                                          _ptr(l2_prefetch), pf_bytes, _stream(stream))
    check("ft2_protect_fused_gemm_ex", st)


def prefill_fused_gemm(x, w, y, bounds_out, workspace, bias=None, seq_offsets=None, num_seqs=None, scale=2.0,
                       correct_nonfinite=True, keys_out=None, nonfinite_count=None, sites=None, n_sites=None,
                       cur_layer=0, base_row=None, gemm_workspace=None, stream=None):
    """ft2_prefill_fused_gemm: y = inject(bf16(x @ w.T + bias)) and, in the same
    kernel's epilogue, ft2_bounds_from_prefill(y, ...) (finalize = 1)."""
    M, K = x.shape
    N = w.shape[0]
    S = num_seqs if num_seqs is not None else (1 if seq_offsets is None else seq_offsets.numel() - 1)
    ns = 0 if sites is None else (n_sites if n_sites is not None else sites.numel() // SITE_BYTES)
    gw = gemm_workspace if gemm_workspace is not None else default_gemm_workspace(x.device)
    st = load().ft2_prefill_fused_gemm(_ptr(x), x.stride(0), _ptr(w), w.stride(0), _ptr(bias), _ptr(y), y.stride(0),
                                       M, N, K, _dtype_of(x), _ptr(seq_offsets), S, float(scale),
                                       int(correct_nonfinite), _ptr(bounds_out), _ptr(keys_out),
                                       _ptr(nonfinite_count), _ptr(sites), ns, cur_layer, _ptr(base_row),
                                       _ptr(workspace), _ptr(gw), gw.numel() * gw.element_size(), _stream(stream))
    check("ft2_prefill_fused_gemm", st)


_GEMM_WS = {}
GEMM_WS_BYTES = 64 << 20   # K-split workspace of the M > 128 kernel (ft2_gemm_workspace_bytes)


def default_gemm_workspace(device) -> torch.Tensor:
    """Per-device zero-filled split-K workspace shared by calls that pass none.
    Created on first use (call once outside CUDA-graph capture); not safe for
    GEMMs running concurrently on different streams -- pass your own then."""
    key = torch.device(device).index if torch.device(device).index is not None else torch.cuda.current_device()
    ws = _GEMM_WS.get(key)
    if ws is None:
        ws = torch.zeros(GEMM_WS_BYTES // 8, dtype=torch.int64, device=torch.device("cuda", key))
        _GEMM_WS[key] = ws
    return ws


def gemm_workspace_bytes(M, N, K) -> int:
    return int(load().ft2_gemm_workspace_bytes(M, N, K))


def make_fault_sites(seed, trial0, n_trials, model, layer_width, n_steps, prompt_len, out=None,
                     layer_uniform=True, step_policy=0, device=None, stream=None, dtype=FT2_BF16):
    """ft2_make_fault_sites -> uint8 tensor [n_trials * 24] (ft2_fault_site records)."""
    widths = (ctypes.c_int32 * len(layer_width))(*[int(v) for v in layer_width])
    g = SiteGeometry(n_steps, prompt_len, len(layer_width), widths, int(layer_uniform), int(step_policy))
    if out is None:
        out = torch.empty(n_trials * SITE_BYTES, dtype=torch.uint8, device=device or "cuda")
    st = load().ft2_make_fault_sites(seed, trial0, n_trials, model, dtype, ctypes.byref(g), _ptr(out),
                                     _stream(stream))
    check("ft2_make_fault_sites", st)
    return out


def inject_faults(y, sites, cur_layer, cur_step, base_row=None, n_sites=None, stream=None):
    t = _as_ft2_tensor(y)
    ns = n_sites if n_sites is not None else sites.numel() // SITE_BYTES
    check("ft2_inject_faults", load().ft2_inject_faults(t, _ptr(sites), ns, cur_layer, cur_step, _ptr(base_row),
                                                        _stream(stream)))


def launch_count() -> int:
    return int(load().ft2_launch_count())


def version() -> str:
    return load().ft2_version().decode()


def allreduce_protect(partial_ptrs, ldp, P, rank, flag_ptrs, words, y, bias=None, mode=FT2_GEMM_CHECK, bounds=None,
                      row_to_seq=None, num_seqs=None, corrected_count=None, sites=None, n_sites=None, cur_layer=0,
                      cur_step=0, base_row=None, stream=None):
    """ft2_allreduce_protect.  partial_ptrs / flag_ptrs: sequences of P
    (peer-mapped) device addresses (host ints); words: device int32 [3]
    (epoch, done, status) of this rank; y: this rank's output."""
    t = _as_ft2_tensor(y)
    S = num_seqs if num_seqs is not None else (bounds.numel() // 2 if bounds is not None else 0)
    ns = 0 if sites is None else (n_sites if n_sites is not None else sites.numel() // SITE_BYTES)
    wp = words.data_ptr()
    if len(partial_ptrs) != P or len(flag_ptrs) != P:
        raise ValueError("allreduce_protect: one partial and one flag pointer per rank")
    pp = (ctypes.c_void_p * P)(*[int(v) for v in partial_ptrs])
    fp = (ctypes.c_void_p * P)(*[int(v) for v in flag_ptrs])
    st = load().ft2_allreduce_protect(pp, int(ldp), int(P), int(rank), fp,
                                      ctypes.c_void_p(wp), ctypes.c_void_p(wp + 4), ctypes.c_void_p(wp + 8), t,
                                      _ptr(bias), int(mode), _ptr(row_to_seq), _ptr(bounds), S,
                                      _ptr(corrected_count), _ptr(sites), ns, cur_layer, cur_step, _ptr(base_row),
                                      _stream(stream))
    check("ft2_allreduce_protect", st)


def ipc_get_handle(t: torch.Tensor):
    """(64-byte handle, byte offset) of the allocation holding t (CUDA IPC)."""
    h = ctypes.create_string_buffer(64)
    off = ctypes.c_uint64(0)
    check("ft2_ipc_get_handle", load().ft2_ipc_get_handle(ctypes.c_void_p(t.data_ptr()), h, ctypes.byref(off)))
    return h.raw, int(off.value)


def ipc_open_handle(handle: bytes) -> int:
    """Map a peer allocation's handle; returns its base device address."""
    p = ctypes.c_void_p(0)
    check("ft2_ipc_open_handle", load().ft2_ipc_open_handle(ctypes.create_string_buffer(handle, 64), ctypes.byref(p)))
    return int(p.value)


def ipc_close(base: int):
    check("ft2_ipc_close", load().ft2_ipc_close(ctypes.c_void_p(base)))


def host_norm(x, w, y, bias=None, eps=1e-5, rms=False, stream=None):
    """Host-model LayerNorm / RMSNorm over the last dim of 2-D x into y
    (include/ft2.h ft2_host_norm; not part of the FT2 method).  Raises
    ValueError when the tensors disagree (dtype, widths, rows): the C ABI only
    sees pointers and leading dimensions."""
    n = x.shape[-1]
    if x.dim() != 2 or y.dim() != 2 or x.stride(-1) != 1 or y.stride(-1) != 1:
        raise ValueError("host_norm: x and y must be 2-D with unit inner stride")
    for name, t in (("w", w), ("bias", bias), ("y", y)):
        if t is not None and t.dtype != x.dtype:
            raise ValueError(f"host_norm: {name} is {t.dtype}, x is {x.dtype}")
    if w.numel() < n or (bias is not None and bias.numel() < n) or y.shape[0] < x.shape[0] or y.shape[1] < n:
        raise ValueError("host_norm: w / bias narrower than x, or y smaller than x")
    check("ft2_host_norm", load().ft2_host_norm(_ptr(x), x.stride(0), _ptr(w), _ptr(bias), _ptr(y), y.stride(0),
                                                x.shape[0], n, float(eps), int(rms), _dtype_of(x), _stream(stream)))
    return y


def host_act(a, y, b=None, act="relu", stream=None):
    """Host-model MLP activation into y: relu(a), or silu(a) * b with
    act="silu_mul" (include/ft2.h ft2_host_act; not part of the FT2 method).
    Raises ValueError when the tensors disagree (dtype, shape)."""
    code = {"relu": 0, "silu_mul": 1}[act]
    if a.dim() != 2 or y.dim() != 2 or a.stride(-1) != 1 or y.stride(-1) != 1:
        raise ValueError("host_act: a and y must be 2-D with unit inner stride")
    if y.dtype != a.dtype or y.shape[0] < a.shape[0] or y.shape[1] < a.shape[1]:
        raise ValueError("host_act: y must match a's dtype and cover its shape")
    if code == 1 and (b is None or b.dim() != 2 or b.dtype != a.dtype or tuple(b.shape) != tuple(a.shape)
                      or b.stride(-1) != 1):
        raise ValueError("host_act: silu_mul needs b with a's dtype and shape")
    check("ft2_host_act", load().ft2_host_act(_ptr(a), a.stride(0), _ptr(b), b.stride(0) if b is not None else 0,
                                              _ptr(y), y.stride(0), a.shape[0], a.shape[-1], code, _dtype_of(a),
                                              _stream(stream)))
    return y
