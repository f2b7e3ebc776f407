"""GPU parity of the fused critical-layer GEMM (tcgen05) against the CPU oracle.

Tolerance (BASELINE.json north_star):
|y_gpu - y_ref| <= 1e-2 * max(|y_ref|, 1e-2 * rms_row(y_ref)) with y_ref the
oracle's fp64-accumulated linear layer (R8) -- fp32 accumulation plus one
bf16 rounding stays far inside it.  Clip masks must be identical on every
non-borderline neuron (|y_ref - b| > 1e-2 |b| for both bounds b), with the
oracle's bounds fed to both sides.

Bit-exact part: the fused epilogue (bias -> RNE -> inject -> check -> count)
must equal the oracle's inject + check applied to the kernel's own PLAIN
output, because PLAIN and CHECK share the deterministic K reduction.
"""
import numpy as np
import pytest
import torch

import ft2_synth
import oracle
from gpu_util import dev, dev_i32, host, sites_to_dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ft2():
    import paper_conf_hpdc_sunzmg00y25_b200 as m
    return m


def _f64(bits):
    import ml_dtypes
    return np.asarray(bits, np.uint16).view(ml_dtypes.bfloat16).astype(np.float64)


def _operands(M, N, K, seed, bias=True):
    x = ft2_synth.gen_bf16((M, K), tau=20, sigma=seed)
    w = ft2_synth.gen_bf16((N, K), tau=21, sigma=seed, scale_log2=ft2_synth.weight_scale_log2(K))
    b = ft2_synth.gen_bf16((N,), tau=22, sigma=seed) if bias else None
    return x, w, b


def _tol_ok(y_gpu_bits, y_ref):
    g = _f64(y_gpu_bits)
    rms = np.sqrt(np.mean(y_ref ** 2, axis=1, keepdims=True))
    tol = 1e-2 * np.maximum(np.abs(y_ref), 1e-2 * rms)
    bad = np.abs(g - y_ref) > tol
    return int(bad.sum()), float(np.max(np.abs(g - y_ref) / np.maximum(np.abs(y_ref), 1e-30)))


def _run(ft2, x, w, b, mode, bounds=None, r2s=None, S=None, sites=None, layer=0, step=0, base_row=None):
    M, N = x.shape[0], w.shape[0]
    xd, wd = dev(x), dev(w)
    bd = None if b is None else dev(b)
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    cnt = torch.zeros(max(S or 1, 1), dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(xd, wd, y, bias=bd, mode=mode, bounds=None if bounds is None else dev(bounds),
                           row_to_seq=None if r2s is None else dev_i32(r2s), num_seqs=S, corrected_count=cnt,
                           sites=None if sites is None else sites_to_dev(sites), cur_layer=layer, cur_step=step,
                           base_row=None if base_row is None else dev_i32(base_row))
    torch.cuda.synchronize()
    return host(y), cnt.cpu().numpy().astype(np.uint32)


GEMM_SHAPES = [
    # (M, N, K)   decode shapes of the configs, ragged tails, prefill tiles
    (1, 768, 768),        # C1: OPT-125m-shaped out_proj, one token
    (16, 768, 768),       # C1 prefill
    (1, 2048, 2048),      # C2 v/out, B = 1
    (32, 2048, 2048),     # C2 v/out, B = 32 (two 16-token tiles, 4-way split)
    (24, 2048, 1792),     # ragged second 16-token tile
    (32, 2048, 8192),     # C2 fc2
    (32, 4096, 4096),     # C3 v / o
    (32, 11008, 4096),    # C3 up
    (32, 4096, 11008),    # C3 down
    (5, 200, 72),         # ragged M, N and K (K % 64 != 0)
    (100, 136, 264),      # M up to 128 (swap-AB, BN = 128)
    (200, 384, 512),      # prefill orientation, ragged M
]


@pytest.mark.parametrize("M,N,K", GEMM_SHAPES)
def test_gemm_plain_within_tolerance(ft2, M, N, K):
    x, w, b = _operands(M, N, K, seed=M + N + K)
    rows = np.arange(M) if M * N * K <= 2 ** 31 else np.unique(np.linspace(0, M - 1, 8).astype(int))
    y_ref, _ = oracle.linear_f64(x[rows], w, b)
    y, _ = _run(ft2, x, w, b, 0)
    nbad, worst = _tol_ok(y[rows], y_ref)
    assert nbad == 0, f"{nbad} elements out of tolerance (worst rel {worst:.3e})"


@pytest.mark.parametrize("M,N,K", [(32, 2048, 2048), (3, 768, 768), (160, 512, 256)])
def test_gemm_plain_vs_cublas(ft2, M, N, K):
    x, w, b = _operands(M, N, K, seed=3)
    y, _ = _run(ft2, x, w, b, 0)
    ref = torch.nn.functional.linear(dev(x).float(), dev(w).float(), dev(b).float()).to(torch.bfloat16)
    d = (torch.from_numpy(_f64(y)) - ref.double().cpu()).abs()
    assert float(d.max()) <= 1e-2 * max(1.0, float(ref.double().abs().max()))


@pytest.mark.parametrize("M,N,K", [(1, 768, 768), (32, 2048, 2048), (24, 2048, 1792), (32, 4096, 11008),
                                   (17, 1000, 136), (200, 384, 512)])
def test_gemm_check_epilogue_bit_exact(ft2, M, N, K):
    x, w, b = _operands(M, N, K, seed=7)
    S = M if M > 1 else 1
    bnds = np.zeros((S, 2), np.uint16)
    rng = np.random.default_rng(M)
    for s in range(S):
        bnds[s] = [oracle.f64_to_bf16(-abs(rng.normal(0.4, 0.2)) - 0.02), oracle.f64_to_bf16(abs(rng.normal(0.4, 0.2)) + 0.02)]
    plain, _ = _run(ft2, x, w, b, 0)
    checked, cnt = _run(ft2, x, w, b, 1, bounds=bnds, S=S)
    ref = plain.copy()
    rc = oracle.protect(ref, bnds, row_to_seq=None if S == 1 else np.arange(M, dtype=np.int32))
    assert np.array_equal(checked, ref)
    assert np.array_equal(cnt, rc)
    assert rc.sum() > 0   # the bounds really clip something


@pytest.mark.parametrize("M,N,K,per_seq", [(32, 4096, 4096, False),
                                           (32, 2048, 2048, True),     # C2 v/out: 16-token tiles, 4-way split
                                           (32, 2048, 8192, True),     # C2 fc2: 12-way split
                                           (32, 4096, 11008, True),    # C3 down
                                           (32, 11008, 4096, True)])   # C3 up
def test_gemm_clip_masks_vs_oracle_non_borderline(ft2, M, N, K, per_seq):
    """R8 mask pin: the GEMM's clip decisions equal the oracle's (fp64 linear ->
    bf16 -> R5 with the same bounds) on every neuron not within 1e-2 relative
    of a bound; per-sequence bounds (row r -> sequence r) at the C2/C3 decode
    shapes, each sequence with its own (lo, hi) around the output's spread."""
    x, w, b = _operands(M, N, K, seed=11 + N + K)
    yd, yb = oracle.linear_f64(x, w, b)
    if per_seq:
        rng = np.random.default_rng(N + K)
        sd = np.std(yd, axis=1)
        S = M
        bnds = np.array([[oracle.f64_to_bf16(-sd[r] * rng.uniform(0.8, 2.5)),
                          oracle.f64_to_bf16(sd[r] * rng.uniform(0.8, 2.5))] for r in range(M)], np.uint16)
        r2s = np.arange(M, dtype=np.int32)
    else:
        S, r2s = 1, None
        bnds = np.array([[oracle.f64_to_bf16(-1.0), oracle.f64_to_bf16(1.0)]], np.uint16)
    ref = yb.copy()
    rc = oracle.protect(ref, bnds, row_to_seq=r2s)
    ref_mask = ref != yb
    checked, cnt = _run(ft2, x, w, b, 1, bounds=bnds, S=S, r2s=r2s)
    plain, _ = _run(ft2, x, w, b, 0)
    gpu_mask = checked != plain
    bf = _f64(bnds)
    lo = bf[(r2s if r2s is not None else np.zeros(M, np.int64)), 0][:, None]
    hi = bf[(r2s if r2s is not None else np.zeros(M, np.int64)), 1][:, None]
    border = (np.abs(yd - lo) <= 1e-2 * np.abs(lo)) | (np.abs(yd - hi) <= 1e-2 * np.abs(hi))
    assert np.array_equal(gpu_mask[~border], ref_mask[~border])
    assert ref_mask.sum() > 100
    # counts agree up to the borderline neurons
    nb_rows = border.sum(axis=1)
    slack = nb_rows if S > 1 else nb_rows.sum()
    assert np.all(np.abs(cnt[:S].astype(np.int64) - rc.astype(np.int64)) <= slack)


@pytest.mark.parametrize("M,N,K", [(32, 2048, 2048), (32, 2048, 8192), (4, 768, 768)])
def test_gemm_l2_prefetch_hint_changes_nothing(ft2, M, N, K):
    """ft2_protect_fused_gemm_ex: the L2 prefetch hint is a hint only --
    outputs and counts are bit-identical with and without it."""
    x, w, b = _operands(M, N, K, seed=23)
    bnds = np.array([[oracle.f64_to_bf16(-0.1), oracle.f64_to_bf16(0.1)]], np.uint16)
    ref, rcnt = _run(ft2, x, w, b, 1, bounds=bnds, S=1)
    nxt = torch.zeros(((3 << 20) + 16) // 2, dtype=torch.bfloat16, device="cuda")   # 3 MB + 16 B
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=1 | 16, bounds=dev(bnds), num_seqs=1,
                           corrected_count=cnt, l2_prefetch=nxt)
    torch.cuda.synchronize()
    assert np.array_equal(host(y), ref) and int(cnt.item()) == int(rcnt[0])


def test_gemm_fault_injection_in_epilogue(ft2):
    M, N, K = 32, 2048, 2048
    x, w, b = _operands(M, N, K, seed=13)
    sites = oracle.make_sites(99, 0, M, oracle.FAULT_EXP, [N] * 4, n_steps=4, prompt_len=1)
    plain, _ = _run(ft2, x, w, b, 0)
    bnds = np.array([[oracle.f64_to_bf16(-4.0), oracle.f64_to_bf16(4.0)]], np.uint16)
    for layer in range(4):
        for step in range(1, 5):
            ref = plain.copy()
            oracle.inject(ref, sites, layer, step)
            inj, _ = _run(ft2, x, w, b, 0, sites=sites, layer=layer, step=step)
            assert np.array_equal(inj, ref)
            rc = oracle.protect(ref, bnds)
            chk, cnt = _run(ft2, x, w, b, 1, bounds=bnds, S=1, sites=sites, layer=layer, step=step)
            assert np.array_equal(chk, ref) and np.array_equal(cnt, rc)


def test_gemm_protected_column_slice(ft2):
    # fused QKV: only the V columns [2N/3, N) are protected
    M, N, K = 8, 3 * 256, 256
    x, w, b = _operands(M, N, K, seed=17)
    bnds = np.array([[oracle.f64_to_bf16(-0.2), oracle.f64_to_bf16(0.2)]], np.uint16)
    plain, _ = _run(ft2, x, w, b, 0)
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=1, bounds=dev(bnds), num_seqs=1,
                           corrected_count=cnt, col_begin=512, col_end=768)
    ref = plain.copy()
    sl = np.ascontiguousarray(ref[:, 512:])
    rc = oracle.protect(sl, bnds)
    ref[:, 512:] = sl
    assert np.array_equal(host(y), ref) and int(cnt.item()) == int(rc[0])


def test_gemm_shared_workspace_across_shapes(ft2):
    """Regression: one workspace serves GEMMs with different tile counts and
    split factors back to back (counters must not be clobbered by partials)."""
    shapes = [(1, 768, 768), (32, 256, 4096), (1, 2048, 2048), (32, 2048, 2048), (8, 4096, 1024), (32, 2048, 2048)]
    for M, N, K in shapes * 2:
        x, w, b = _operands(M, N, K, seed=M * 3 + N)
        y, _ = _run(ft2, x, w, b, 0)
        yr, _ = oracle.linear_f64(x, w, b)
        nbad, worst = _tol_ok(y, yr)
        assert nbad == 0, (M, N, K, nbad, worst)


def _directed_sites(n_sites, cols, step=1, layer=0, token=0):
    """n_sites sites, all at (step, layer), columns `cols`; with base_row = 0
    every one lands in row 0 (+ token during the prefill): a dense, directed
    site set that overflows any per-CTA site list."""
    s = np.zeros(n_sites, oracle.SITE_DTYPE)
    s["trial"] = np.arange(n_sites)
    s["step"], s["layer"], s["token"] = step, layer, token
    s["col"] = cols
    s["xor_mask"] = 1 << (np.arange(n_sites) % 16)
    s["nbits"] = 1
    return s


@pytest.mark.parametrize("M,N,K,step", [(32, 256, 256, 1), (8, 2048, 512, 3), (200, 512, 256, 0)])
def test_gemm_site_overflow_is_never_dropped(ft2, M, N, K, step):
    """more sites than the per-CTA (decode: 64) or per-row-per-tile
    (prefill: 4) lists hold -- here 100 sites in one row and one 128/256-wide
    tile -- must still all be applied, exactly as the oracle's R7 applies them."""
    x, w, b = _operands(M, N, K, seed=29)
    plain, _ = _run(ft2, x, w, b, 0)
    sites = _directed_sites(100, (np.arange(100) * 7) % 128, step=step, token=1 if step == 0 else 0)
    base = np.zeros(100, np.int32)
    ref = plain.copy()
    oracle.inject(ref, sites, 0, step, base_row=base)
    assert int((ref != plain).sum()) >= 90      # the flips really land (a few columns repeat and cancel)
    inj, _ = _run(ft2, x, w, b, 0, sites=sites, layer=0, step=step, base_row=base)
    assert np.array_equal(inj, ref)
    bnds = np.array([[oracle.f64_to_bf16(-0.5), oracle.f64_to_bf16(0.5)]], np.uint16)
    rc = oracle.protect(ref, bnds)
    chk, cnt = _run(ft2, x, w, b, 1, bounds=bnds, S=1, sites=sites, layer=0, step=step, base_row=base)
    assert np.array_equal(chk, ref) and np.array_equal(cnt, rc)


@pytest.mark.parametrize("env", [{"FT2_GEMM_BA": "64"}, {"FT2_GEMM_BA": "128"},
                                 {"FT2_GEMM_BA": "64", "FT2_GEMM_XMC": "1"},
                                 {"FT2_GEMM_BA": "128", "FT2_GEMM_BN": "16"},
                                 {"FT2_GEMM_MMA2": "0"},                      # one MMA issuer (round 1)
                                 {"FT2_GEMM_BA": "128", "FT2_GEMM_BN": "32", "FT2_GEMM_MMA2": "2"},   # 128-row MMA2
                                 {"FT2_GEMM_TRIGGER": "1"}, {"FT2_GEMM_TRIGGER": "2"}])
def test_gemm_tile_variants_in_subprocess(env):
    """The 64- and 128-row feature tiles and the opt-in x multicast (planner
    knobs read once per process) give results within R8's tolerance and
    epilogues bit-exact with the oracle applied to their own PLAIN output."""
    import os
    import subprocess
    import sys
    code = r'''
import numpy as np, torch, sys
sys.path[:0] = [ROOT, ROOT + "/tests"]
import oracle, ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
from gpu_util import dev, host
for M, N, K in ((32, 2048, 2048), (16, 1024, 512), (32, 4096, 4096), (8, 640, 2304), (27, 2048, 1000), (3, 512, 72)):
    x = ft2_synth.gen_bf16((M, K), 20, 5); w = ft2_synth.gen_bf16((N, K), 21, 5, scale_log2=ft2_synth.weight_scale_log2(K))
    b = ft2_synth.gen_bf16((N,), 22, 5)
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=0)
    torch.cuda.synchronize(); plain = host(y)
    yd, _ = oracle.linear_f64(x, w, b)
    g = plain.astype(np.uint32) << 16
    gv = g.view(np.float32).astype(np.float64)
    rms = np.sqrt(np.mean(yd ** 2, axis=1, keepdims=True))
    assert np.all(np.abs(gv - yd) <= 1e-2 * np.maximum(np.abs(yd), 1e-2 * rms)), (M, N, K)
    bnd = np.array([[oracle.f64_to_bf16(-0.05), oracle.f64_to_bf16(0.05)]], np.uint16)
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=1, bounds=dev(bnd), num_seqs=1, corrected_count=cnt)
    torch.cuda.synchronize()
    ref = plain.copy(); rc = oracle.protect(ref, bnd)
    assert np.array_equal(host(y), ref) and int(cnt.item()) == int(rc[0]), (M, N, K)
print("ok")
'''.replace("ROOT", repr(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
    r = subprocess.run([sys.executable, "-c", code], env={**os.environ, **env}, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-3000:]
