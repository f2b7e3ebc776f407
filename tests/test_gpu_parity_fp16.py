"""FP16 (the paper's own precision) through every kernel: bounds,
prefill correction, check-and-clip, injection and the fused tcgen05 GEMM --
bit-exact against the oracle's FP16 path (GEMM: tolerance + bit-exact epilogue)."""
import numpy as np
import pytest
import torch

import ft2_synth
import oracle
from gpu_util import dev_i32, sites_to_dev

pytestmark = pytest.mark.gpu
F16 = oracle.DT_FP16


@pytest.fixture(scope="module")
def ft2():
    import paper_conf_hpdc_sunzmg00y25_b200 as m
    return m


def devh(a):
    return torch.from_numpy(np.ascontiguousarray(a, np.uint16).view(np.int16)).view(torch.float16).cuda()


def hosth(t):
    return t.contiguous().cpu().view(torch.int16).numpy().view(np.uint16)


def _fp16(rows, n, seed, scale_log2=0, edges=True):
    b = ft2_synth.gen_bf16((rows, n), 5, seed, scale_log2=scale_log2)
    y = torch.from_numpy(b.view(np.int16)).view(torch.bfloat16).float().half().view(torch.int16).numpy().view(np.uint16).copy()
    if edges:
        e = np.array([0x7E00, 0xFE01, 0x7C01, 0x7C00, 0xFC00, 0x0000, 0x8000, 0x0001, 0x7BFF, 0xFBFF], np.uint16)
        flat = y.reshape(-1)
        idx = np.arange(7, flat.size, 173)
        flat[idx] = e[np.arange(idx.size) % e.size]
    return y


@pytest.mark.parametrize("shape,so", [((16, 768), None), ((512, 4096), list(range(0, 513, 64))),
                                      ((6, 4096), [0, 1, 2, 3, 4, 5, 6])])
def test_fp16_bounds_and_correction(ft2, shape, so):
    y = _fp16(*shape, seed=shape[0])
    if shape[0] == 6:
        y[0, :] = 0x7E00; y[4, :] = 0xFC00       # all-NaN sequence, patch-list overflow
    ref = y.copy()
    rb, rk, rnf = oracle.bounds(ref, seq_offsets=so, correct_nonfinite=True, dtype=F16)
    S = 1 if so is None else len(so) - 1
    yd = devh(y)
    b = torch.zeros((S, 2), dtype=torch.float16, device="cuda")
    nf = torch.zeros(S, dtype=torch.int32, device="cuda")
    nv = torch.zeros(S, dtype=torch.int32, device="cuda")
    rnv = oracle.nan_vulnerable_count(y, seq_offsets=so, dtype=F16)
    ft2.bounds_from_prefill(yd, b, ft2.make_workspace(S), seq_offsets=None if so is None else dev_i32(so),
                            num_seqs=S, correct_nonfinite=True, nonfinite_count=nf, nan_vulnerable_count=nv)
    assert np.array_equal(hosth(b), rb) and np.array_equal(hosth(yd), ref)
    assert np.array_equal(nv.cpu().numpy().astype(np.uint32), rnv)
    assert np.array_equal(nf.cpu().numpy().astype(np.uint32), rnf)


@pytest.mark.parametrize("rows,n", [(1, 8), (32, 2048), (129, 4096)])
def test_fp16_protect(ft2, rows, n):
    y = _fp16(rows, n, seed=n)
    bnd = np.array([[0xB800, 0x3A00]], np.uint16)
    ref = y.copy()
    rc = oracle.protect(ref, bnd, dtype=F16)
    yd = devh(y)
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect(yd, devh(bnd), corrected_count=cnt)
    assert np.array_equal(hosth(yd), ref) and int(cnt.item()) == int(rc[0])


def test_fp16_sites_and_inject(ft2):
    w = [2048] * 6
    for model in (0, 1, 2):
        ref = oracle.make_sites(3, 0, 1000, model, w, 8, 4, dtype=F16)
        got = ft2.make_fault_sites(3, 0, 1000, model, w, 8, 4, dtype=1)
        assert got.cpu().numpy().tobytes() == ref.tobytes()
    e = oracle.make_sites(3, 0, 1000, 2, w, 8, 4, dtype=F16)
    assert np.all((e["xor_mask"] & 0x7C00) == e["xor_mask"])   # FP16 exponent bits 10..14


@pytest.mark.parametrize("M,N,K", [(1, 768, 768), (32, 2048, 2048), (32, 4096, 4096), (200, 384, 512)])
def test_fp16_fused_gemm(ft2, M, N, K):
    x = _fp16(M, K, 20, edges=False)
    w = _fp16(N, K, 21, scale_log2=ft2_synth.weight_scale_log2(K), edges=False)
    bias = _fp16(1, N, 22, edges=False).reshape(-1)
    yd_f64, _ = oracle.linear_f64(x, w, bias, dtype=F16)
    plain = torch.empty((M, N), dtype=torch.float16, device="cuda")
    ft2.protect_fused_gemm(devh(x), devh(w), plain, bias=devh(bias), mode=0)
    g = hosth(plain).view(np.float16).astype(np.float64)
    tol = 1e-2 * np.maximum(np.abs(yd_f64), 1e-2 * np.sqrt(np.mean(yd_f64 ** 2, axis=1, keepdims=True)))
    assert np.all(np.abs(g - yd_f64) <= tol)
    bnd = np.array([[0xB666, 0x3666]], np.uint16)   # +-0.4
    chk = torch.empty((M, N), dtype=torch.float16, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(devh(x), devh(w), chk, bias=devh(bias), mode=1, bounds=devh(bnd), num_seqs=1,
                           corrected_count=cnt)
    ref = hosth(plain).copy()
    rc = oracle.protect(ref, bnd, dtype=F16)
    assert np.array_equal(hosth(chk), ref) and int(cnt.item()) == int(rc[0]) and rc[0] > 0
