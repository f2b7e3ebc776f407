"""Pins for the oracle's representation layer (R0) -- CPU only.

Pinned against: IEEE bf16 semantics via numpy/ml_dtypes (independent
libraries), PAPER.md L185 (layout + NaN definition).
"""
import math

import ml_dtypes
import numpy as np
import pytest

import oracle

ALL = np.arange(65536, dtype=np.uint32).astype(np.uint16)


def _f(b):
    return ALL[b:b + 1].view(ml_dtypes.bfloat16).astype(np.float64)[0] if isinstance(b, int) else None


def test_isnan_isinf_match_numpy_for_all_patterns():
    vals = ALL.view(ml_dtypes.bfloat16).astype(np.float32)
    for b in range(0, 65536, 1):
        assert oracle.isnan(b) == bool(np.isnan(vals[b]))
        assert oracle.isinf(b) == bool(np.isinf(vals[b]))


def test_key_is_total_order_on_non_nan_and_roundtrips():
    vals = ALL.view(ml_dtypes.bfloat16).astype(np.float64)
    keys = np.array([oracle.key(int(b)) for b in ALL], dtype=np.int64)
    for b in range(65536):
        assert oracle.unkey(int(keys[b])) == b
    nonnan = ~np.isnan(vals)
    # sort non-NaN patterns by key: values must be non-decreasing, and the only
    # equal-value neighbours are (-0, +0) in that order (reading A7).
    idx = np.nonzero(nonnan)[0]
    order = idx[np.argsort(keys[idx])]
    v = vals[order]
    assert np.all(np.diff(v) >= 0)
    ties = np.nonzero(np.diff(v) == 0)[0]
    assert len(ties) == 1 and ALL[order[ties[0]]] == 0x8000 and ALL[order[ties[0] + 1]] == 0x0000
    # NaN keys fall strictly outside [key(-Inf), key(+Inf)] = [0x007F, 0xFF80]
    assert oracle.key(0xFF80) == 0x007F and oracle.key(0x7F80) == 0xFF80
    nk = keys[~nonnan]
    assert np.all((nk < 0x007F) | (nk > 0xFF80))


def test_rne_matches_ml_dtypes_on_fp32_inputs():
    rng = np.random.default_rng(0)
    bits = rng.integers(0, 2**32, size=20000, dtype=np.uint64).astype(np.uint32)
    # add every halfway/odd-even case around a few binades plus extremes
    extra = []
    for hi in [0x3F80, 0x3F81, 0x7F7F, 0x0000, 0x0001, 0x007F, 0x0080, 0x8001, 0xFF7F, 0x7F7E]:
        for lo in [0x0000, 0x7FFF, 0x8000, 0x8001, 0xFFFF]:
            extra.append((hi << 16) | lo)
    bits = np.concatenate([bits, np.array(extra, dtype=np.uint32)])
    f = bits.view(np.float32)
    f = f[~np.isnan(f)]
    want = f.astype(ml_dtypes.bfloat16).view(np.uint16)
    for x, w in zip(f, want):
        assert oracle.f64_to_bf16(float(x)) == int(w), hex(int(np.float32(x).view(np.uint32)))


def test_rne_of_doubles_is_nearest():
    # from fp64 the oracle must pick the nearest bf16 (no double rounding via fp32)
    rng = np.random.default_rng(1)
    for _ in range(3000):
        d = float(rng.standard_normal() * 10.0 ** rng.integers(-40, 38))
        r = oracle.f64_to_bf16(d)
        rv = oracle.bf16_to_f64(r)
        up = oracle.unkey(oracle.key(r) + 1)
        dn = oracle.unkey(oracle.key(r) - 1)
        for nb in (up, dn):
            nv = oracle.bf16_to_f64(nb)
            if math.isfinite(nv):
                assert abs(rv - d) <= abs(nv - d)
    # a double just above a bf16 halfway point rounds up, though via fp32 it would tie
    half = 1.0 + 2.0 ** -8
    assert oracle.f64_to_bf16(half) == 0x3F80           # tie -> even
    assert oracle.f64_to_bf16(half + 2.0 ** -40) == 0x3F81


def test_directed_rounding_brackets_value():
    rng = np.random.default_rng(2)
    for _ in range(3000):
        d = float(rng.standard_normal() * 10.0 ** rng.integers(-40, 38))
        lo = oracle.f64_to_bf16_dir(d, -1)
        hi = oracle.f64_to_bf16_dir(d, +1)
        assert oracle.bf16_to_f64(lo) <= d <= oracle.bf16_to_f64(hi)
        assert oracle.key(hi) - oracle.key(lo) in (0, 1) or (d == 0.0)
