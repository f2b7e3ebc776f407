"""Seeded synthetic inputs (SURVEY.md §8(d) "Synthetic input generator").

This module is the ONLY code shared by the CPU oracle side (``oracle/``, tests)
and the GPU side (``bench.py``, GPU parity tests).  It holds none of FT2's
arithmetic: no order keys, no bounds, no clipping, no fault sites.  It only
produces bf16 bit patterns (as ``uint16``) from a counter-based generator so
that both sides see identical tensors.

Recipe (exact integer construction):

* element ``i`` of tensor ``tau`` under seed ``sigma``:
  ``(u0,u1,u2,u3) = Philox4x32-10(ctr=(i_lo, i_hi, tau, 0x47454E00), key=(sigma_lo, sigma_hi))``
* ``z = (u0>>16) + (u0&0xFFFF) + (u1>>16) + (u1&0xFFFF) - 131070``  (Irwin-Hall(4))
* ``v = z * 2**-17`` (exact in fp32; sigma ~0.289, most values in (-1, 1) as
  PAPER.md L202 reports for critical layers)
* outlier iff ``(u2 & 0x3FF) == 0`` (p = 2**-10): ``v *= 2**(5 + ((u2>>10)&3))``
  -- the "few large values" of PAPER.md L261 / Fig 12
* ``y = RNE_bf16(v)``; optional ``scale_log2`` multiplies v by 2**scale_log2
  first (exact), used for GEMM weights (``-ceil(log2 sqrt K)``).

Two implementations of the same recipe: numpy on the host (``gen_bf16``) and
torch int64 ops on any device (``gen_bf16_torch``) for tensors too large to
build on the host quickly.  ``tests/test_synth.py`` checks they agree.
"""
from __future__ import annotations

import math

import numpy as np

__all__ = ["philox4x32_10_np", "gen_bf16", "gen_bf16_torch", "weight_scale_log2",
           "plant_edge_values", "GEN_TAG"]

GEN_TAG = 0x47454E00  # "GEN\0"

_M0 = np.uint64(0xD2511F53)
_M1 = np.uint64(0xCD9E8D57)
_W0 = 0x9E3779B9
_W1 = 0xBB67AE85
_MASK32 = np.uint64(0xFFFFFFFF)


def philox4x32_10_np(c0, c1, c2, c3, k0: int, k1: int):
    """Vectorised Philox4x32-10 (Salmon et al., SC'11) on uint64-held 32-bit lanes."""
    c0 = np.asarray(c0, dtype=np.uint64) & _MASK32
    c1 = np.broadcast_to(np.asarray(c1, dtype=np.uint64), c0.shape) & _MASK32
    c2 = np.broadcast_to(np.asarray(c2, dtype=np.uint64), c0.shape) & _MASK32
    c3 = np.broadcast_to(np.asarray(c3, dtype=np.uint64), c0.shape) & _MASK32
    key0, key1 = k0 & 0xFFFFFFFF, k1 & 0xFFFFFFFF
    for r in range(10):
        if r:
            key0 = (key0 + _W0) & 0xFFFFFFFF
            key1 = (key1 + _W1) & 0xFFFFFFFF
        p0 = _M0 * c0
        p1 = _M1 * c2
        hi0, lo0 = p0 >> np.uint64(32), p0 & _MASK32
        hi1, lo1 = p1 >> np.uint64(32), p1 & _MASK32
        c0, c1, c2, c3 = (hi1 ^ c1 ^ np.uint64(key0)), lo1, (hi0 ^ c3 ^ np.uint64(key1)), lo0
    return c0, c1, c2, c3


def _rne_f32_to_bf16_bits(v: np.ndarray) -> np.ndarray:
    """Round fp32 -> bf16 (nearest-even) on bit patterns; v is finite here."""
    b = v.astype(np.float32).view(np.uint32).astype(np.uint64)
    lsb = (b >> np.uint64(16)) & np.uint64(1)
    r = (b + np.uint64(0x7FFF) + lsb) >> np.uint64(16)
    return (r & np.uint64(0xFFFF)).astype(np.uint16)


def weight_scale_log2(K: int) -> int:
    """GEMM weights are scaled by 2**-ceil(log2 sqrt K)."""
    return -int(math.ceil(math.log2(math.sqrt(K))))


def gen_bf16(shape, tau: int, sigma: int, scale_log2: int = 0, start: int = 0, outliers: bool = True) -> np.ndarray:
    """bf16 bit patterns (uint16 array of ``shape``) for tensor id ``tau``, seed ``sigma``.

    Element ``i`` is the row-major flat index offset by ``start``.  outliers=False
    drops the planted 2**-10 outliers (every value keeps its bulk draw).
    """
    n = int(np.prod(shape)) if len(shape) else 1
    i = np.arange(start, start + n, dtype=np.uint64)
    u0, u1, u2, _ = philox4x32_10_np(i & _MASK32, i >> np.uint64(32), tau, GEN_TAG,
                                     sigma & 0xFFFFFFFF, (sigma >> 32) & 0xFFFFFFFF)
    z = ((u0 >> np.uint64(16)) + (u0 & np.uint64(0xFFFF)) + (u1 >> np.uint64(16))
         + (u1 & np.uint64(0xFFFF))).astype(np.int64) - 131070
    e = np.where((u2 & np.uint64(0x3FF)) == 0, 5 + ((u2 >> np.uint64(10)) & np.uint64(3)).astype(np.int64), 0)
    if not outliers:
        e = np.zeros_like(e)
    v = np.ldexp(z.astype(np.float64), (e - 17 + scale_log2).astype(np.int32)).astype(np.float32)
    return _rne_f32_to_bf16_bits(v).reshape(shape)


def gen_bf16_torch(shape, tau: int, sigma: int, scale_log2: int = 0, device="cpu", start: int = 0,
                   outliers: bool = True):
    """Same recipe as :func:`gen_bf16`, built with torch int64 ops on ``device``.

    Returns a ``torch.bfloat16`` tensor.  Chunked to bound temporary memory.
    """
    import torch

    n = 1
    for s in shape:
        n *= int(s)
    out = torch.empty(n, dtype=torch.int16, device=device)
    M32 = 0xFFFFFFFF
    chunk = 1 << 26
    for off in range(0, n, chunk):
        m = min(chunk, n - off)
        i = torch.arange(start + off, start + off + m, dtype=torch.int64, device=device)
        c0 = i & M32
        c1 = i >> 32
        c2 = torch.full_like(c0, tau & M32)
        c3 = torch.full_like(c0, GEN_TAG)
        k0, k1 = sigma & M32, (sigma >> 32) & M32
        for r in range(10):
            if r:
                k0 = (k0 + _W0) & M32
                k1 = (k1 + _W1) & M32
            # 32x32 -> 64 multiply split into 16-bit halves to stay inside int64
            hi0, lo0 = _mulhilo32_t(0xD2511F53, c0)
            hi1, lo1 = _mulhilo32_t(0xCD9E8D57, c2)
            c0, c1, c2, c3 = (hi1 ^ c1 ^ k0), lo1, (hi0 ^ c3 ^ k1), lo0
        u0, u1, u2 = c0, c1, c2
        z = (u0 >> 16) + (u0 & 0xFFFF) + (u1 >> 16) + (u1 & 0xFFFF) - 131070
        e = torch.where((u2 & 0x3FF) == 0, 5 + ((u2 >> 10) & 3), torch.zeros_like(u2))
        if not outliers:
            e = torch.zeros_like(u2)
        v = z.to(torch.float64) * torch.pow(2.0, (e - 17 + scale_log2).to(torch.float64))
        b = v.to(torch.float32).view(torch.int32).to(torch.int64) & M32
        lsb = (b >> 16) & 1
        r16 = ((b + 0x7FFF + lsb) >> 16) & 0xFFFF
        out[off:off + m] = (r16 - ((r16 >> 15) << 16)).to(torch.int16)
    return out.view(torch.bfloat16).reshape(tuple(shape))


def _mulhilo32_t(a: int, x):
    """(hi, lo) 32-bit halves of a*x for 32-bit unsigned a, x held in int64."""
    a_lo, a_hi = a & 0xFFFF, a >> 16
    x_lo, x_hi = x & 0xFFFF, x >> 16
    ll = a_lo * x_lo
    lh = a_lo * x_hi
    hl = a_hi * x_lo
    hh = a_hi * x_hi
    mid = (ll >> 16) + (lh & 0xFFFF) + (hl & 0xFFFF)
    lo = ((mid & 0xFFFF) << 16) | (ll & 0xFFFF)
    hi = hh + (lh >> 16) + (hl >> 16) + (mid >> 16)
    return hi & 0xFFFFFFFF, lo & 0xFFFFFFFF


# Edge corpus (SURVEY.md §8(d) last bullet): NaN of both signs with varied
# payloads, +-Inf, +-0, subnormals and +-max planted at fixed strides.
EDGE_VALUES = np.array([
    0x7FC0, 0xFFC0, 0x7F81, 0xFFFF, 0x7FFF, 0xFF81,   # NaNs
    0x7F80, 0xFF80,                                   # +-Inf
    0x0000, 0x8000,                                   # +-0
    0x0001, 0x807F, 0x0040,                           # subnormals
    0x7F7F, 0xFF7F,                                   # +-max finite
], dtype=np.uint16)


def plant_edge_values(y: np.ndarray, stride: int = 97, offset: int = 13) -> np.ndarray:
    """Return a copy of flat bf16 bits ``y`` with EDGE_VALUES planted every ``stride``."""
    out = np.array(y, dtype=np.uint16, copy=True)
    flat = out.reshape(-1)
    idx = np.arange(offset, flat.size, stride)
    flat[idx] = EDGE_VALUES[np.arange(idx.size) % EDGE_VALUES.size]
    return out
