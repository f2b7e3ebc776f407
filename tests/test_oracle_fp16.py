"""Pins for the oracle's FP16 path (the paper's main precision, PAPER.md L282;
layout 1/5/10, L185).  Independent references: numpy float16 (IEEE binary16
conversions and classification), CPU torch float16 clamp/nan_to_num
(L272) and amin/amax, the Fig. 7 closed forms."""
import numpy as np
import pytest
import torch

import ft2_synth
import oracle

F16 = oracle.DT_FP16
ALL = np.arange(65536, dtype=np.uint32).astype(np.uint16)


def test_fp16_classification_and_values_match_numpy():
    v = ALL.view(np.float16).astype(np.float64)
    for b in range(0, 65536, 7):
        assert oracle.isnan_dt(b, F16) == bool(np.isnan(v[b]))
        assert oracle.isinf_dt(b, F16) == bool(np.isinf(v[b]))
        if not np.isnan(v[b]):
            assert oracle.to_f64(b, F16) == v[b]


def test_fp16_rne_matches_numpy():
    rng = np.random.default_rng(0)
    f32 = rng.integers(0, 2 ** 32, 20000, dtype=np.uint64).astype(np.uint32).view(np.float32)
    f32 = f32[np.isfinite(f32)]
    for x in f32:
        assert oracle.f64_to(float(x), F16) == int(np.float32(x).astype(np.float16).view(np.uint16))
    d = rng.standard_normal(5000) * 10.0 ** rng.integers(-9, 6, 5000)
    for x in d:   # numpy's double -> half conversion is correctly rounded
        assert oracle.f64_to(float(x), F16) == int(np.float64(x).astype(np.float16).view(np.uint16))
    # ties to even at 1 + 2^-11 and overflow to Inf above 65520
    assert oracle.f64_to(1.0 + 2.0 ** -11, F16) == 0x3C00
    assert oracle.f64_to(65519.9, F16) == 0x7BFF and oracle.f64_to(65520.0, F16) == 0x7C00


def test_fp16_scale_closed_form_and_saturation():
    for raw in (0x3C00, 0xBC00, 0x3555, 0xC200, 0x0001, 0x8001):
        v = oracle.to_f64(raw, F16)
        if v >= 0:
            assert oracle.to_f64(oracle.scale_bound(raw, 2.0, True, F16), F16) == 2 * v
        if v <= 0:
            assert oracle.to_f64(oracle.scale_bound(raw, 2.0, False, F16), F16) == 2 * v
    assert oracle.scale_bound(0x7BFF, 2.0, True, F16) == 0x7BFF      # 65504 * 2 saturates (A8)
    assert oracle.scale_bound(0xFBFF, 2.0, False, F16) == 0xFBFF


def _fp16_tensor(rows, n, seed):
    # bf16 generator values re-expressed in fp16 (exactly representable for the bulk)
    b = ft2_synth.gen_bf16((rows, n), 5, seed)
    f = torch.from_numpy(b.view(np.int16)).view(torch.bfloat16).float().half()
    y = f.view(torch.int16).numpy().view(np.uint16).copy()
    edges = np.array([0x7E00, 0xFE01, 0x7C01, 0x7C00, 0xFC00, 0x0000, 0x8000, 0x0001, 0x7BFF, 0xFBFF], np.uint16)
    flat = y.reshape(-1)
    idx = np.arange(3, flat.size, 41)
    flat[idx] = edges[np.arange(idx.size) % edges.size]
    return y


@pytest.mark.parametrize("seed", [1, 2])
def test_fp16_protect_vs_torch(seed):
    y = _fp16_tensor(24, 160, seed)
    lo, hi = 0xB800, 0x3A00   # -0.5, 0.75
    out = y.copy()
    cnt = oracle.protect(out, np.array([[lo, hi]], np.uint16), dtype=F16)
    t = torch.from_numpy(y.view(np.int16)).view(torch.float16)
    ref = torch.clamp(torch.nan_to_num(t, nan=0.0), -0.5, 0.75).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(out, ref) and cnt[0] == int((out != y).sum())


def test_fp16_bounds_vs_torch_and_correction():
    y = _fp16_tensor(20, 96, 3)
    b, k, nf = oracle.bounds(y.copy(), scale=1.0, dtype=F16)
    t = torch.from_numpy(y.view(np.int16)).view(torch.float16).float()
    fin = torch.isfinite(t)
    assert oracle.to_f64(oracle.unkey(int(k[0, 0])), F16) == t[fin].amin().item()
    assert oracle.to_f64(oracle.unkey(int(k[0, 1])), F16) == t[fin].amax().item()
    assert nf[0] == int((~fin).sum())
    y2 = y.copy()
    b2, _, _ = oracle.bounds(y2, scale=2.0, correct_nonfinite=True, dtype=F16)
    assert not np.any((y2 & 0x7C00) == 0x7C00)
    f = (y & 0x7C00) != 0x7C00
    assert np.array_equal(y2[f], y[f])


def test_fig7_fp16_exponent_msb():
    # PAPER.md L185 / Fig. 7 in the paper's own FP16 layout: (1,2) -> NaN, 0.5 -> 32768
    v = ALL.view(np.float16).astype(np.float64)
    vuln = ALL[((v > 1) & (v < 2)) | ((v < -1) & (v > -2))]
    for b in vuln[::13]:
        assert oracle.isnan_dt(int(b) ^ 0x4000, F16)
    assert oracle.to_f64(0x3800 ^ 0x4000, F16) == 32768.0
