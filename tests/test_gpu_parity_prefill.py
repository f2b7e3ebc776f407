"""GPU parity of the prefill-shaped critical layer (persistent 128x256 tcgen05
kernel) and of ft2_prefill_fused_gemm, the first-token bound derivation fused
into its epilogue.

* PLAIN / CHECK at M > 128 against the oracle's fp64 linear layer (R8, the
  GEMM tolerance of DESIGN.md) and the bit-exact check epilogue.
* DERIVE: bounds, raw keys, non-finite counts and the corrected layer output
  must be bit-identical to the oracle's R2-R4 (oracle.bounds with
  correct_nonfinite) applied to the kernel's own PLAIN output -- PLAIN and
  DERIVE share the K reduction, so the comparison isolates the fused part.
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
    x = ft2_synth.gen_bf16((M, K), tau=30, sigma=seed)
    w = ft2_synth.gen_bf16((N, K), tau=31, sigma=seed, scale_log2=ft2_synth.weight_scale_log2(K))
    b = ft2_synth.gen_bf16((N,), tau=32, sigma=seed) if bias else None
    return x, w, b


def _plain(ft2, x, w, b, sites=None, layer=0, base_row=None):
    M, N = x.shape[0], w.shape[0]
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=None if b is None else dev(b), mode=0,
                           sites=None if sites is None else sites_to_dev(sites), cur_layer=layer, cur_step=0,
                           base_row=None if base_row is None else dev_i32(base_row))
    torch.cuda.synchronize()
    return host(y)


def _derive(ft2, x, w, b, so=None, S=1, correct=True, sites=None, layer=0, ws=None, scale=2.0):
    M, N = x.shape[0], w.shape[0]
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    bnd = torch.zeros((S, 2), dtype=torch.bfloat16, device="cuda")
    keys = torch.zeros((S, 2), dtype=torch.int32, device="cuda")
    nf = torch.zeros(S, dtype=torch.int32, device="cuda")
    ws = ft2.make_workspace(S) if ws is None else ws
    sod = None if so is None else dev_i32(so)
    ft2.prefill_fused_gemm(dev(x), dev(w), y, bnd, ws, bias=None if b is None else dev(b), seq_offsets=sod,
                           num_seqs=S, scale=scale, correct_nonfinite=correct, keys_out=keys, nonfinite_count=nf,
                           sites=None if sites is None else sites_to_dev(sites), cur_layer=layer, base_row=sod)
    torch.cuda.synchronize()
    return host(y), host(bnd), keys.cpu().numpy(), nf.cpu().numpy().astype(np.uint32), ws


PREFILL_SHAPES = [
    (4096, 2048, 2048),   # C2 prefill (B = 32 x 128 tokens), OPT-1.3B v / out_proj
    (512, 4096, 4096),    # C3 prefill (B = 32 x 16 tokens), Llama-2-7B v / o
    (512, 11008, 4096),   # C3 up_proj: N % 256 != 0
    (300, 520, 200),      # ragged M, N (N % 256 != 0) and K (K % 64 != 0)
    (129, 256, 64),       # one row past the decode orientation
]


@pytest.mark.parametrize("M,N,K", PREFILL_SHAPES)
def test_prefill_plain_within_tolerance(ft2, M, N, K):
    x, w, b = _operands(M, N, K, seed=M + N)
    rows = np.arange(M) if M * N * K <= 2 ** 31 else np.unique(np.linspace(0, M - 1, 12).astype(int))
    y = _plain(ft2, x, w, b)
    y_ref, _ = oracle.linear_f64(x[rows], w, b)
    g = _f64(y[rows])
    rms = np.sqrt(np.mean(y_ref ** 2, axis=1, keepdims=True))
    bad = np.abs(g - y_ref) > 1e-2 * np.maximum(np.abs(y_ref), 1e-2 * rms)
    assert int(bad.sum()) == 0


def test_prefill_check_epilogue_bit_exact(ft2):
    M, N, K = 384, 768, 512
    x, w, b = _operands(M, N, K, seed=5)
    S = 3
    r2s = (np.arange(M) // 128).astype(np.int32)
    bnds = np.array([[oracle.f64_to_bf16(-0.3), oracle.f64_to_bf16(0.3)],
                     [oracle.f64_to_bf16(-0.5), oracle.f64_to_bf16(0.2)],
                     [oracle.f64_to_bf16(0.01), oracle.f64_to_bf16(0.9)]], np.uint16)
    plain = _plain(ft2, x, w, b)
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    cnt = torch.zeros(S, dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=1, bounds=dev(bnds), row_to_seq=dev_i32(r2s),
                           num_seqs=S, corrected_count=cnt)
    ref = plain.copy()
    rc = oracle.protect(ref, bnds, row_to_seq=r2s)
    assert np.array_equal(host(y), ref)
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), rc) and rc.sum() > 0


def _tp_keys(rk):
    """oracle raw keys (key(min), key(max)) -> the keys_out encoding of include/ft2.h
    (0xFFFF - key(min), key(max)), -1 for a sequence without a finite value."""
    k = rk.astype(np.int64).copy()
    k[:, 0] = np.where(rk[:, 0] >= 0, 0xFFFF - rk[:, 0], -1)
    return k.astype(np.int32)


def _check_derive(ft2, x, w, b, so, S, sites=None, layer=0, scale=2.0):
    plain = _plain(ft2, x, w, b, sites=sites, layer=layer, base_row=so)
    ref = plain.copy()
    rb, rk, rnf = oracle.bounds(ref, seq_offsets=so, scale=scale, correct_nonfinite=True)
    y, bnd, keys, nf, ws = _derive(ft2, x, w, b, so=so, S=S, sites=sites, layer=layer, scale=scale)
    assert np.array_equal(bnd, rb)
    assert np.array_equal(keys, _tp_keys(rk))
    assert np.array_equal(nf, rnf)
    assert np.array_equal(y, ref)
    # the workspace is left zeroed (self-cleaning protocol of ft2_bounds_from_prefill)
    assert int(ws.abs().sum().item()) == 0
    return rnf


@pytest.mark.parametrize("M,N,K,S", [(4096, 2048, 2048, 32), (512, 4096, 4096, 32), (512, 11008, 4096, 32),
                                     (300, 520, 200, 3), (256, 256, 128, 1)])
def test_prefill_derive_bit_exact(ft2, M, N, K, S):
    x, w, b = _operands(M, N, K, seed=K + S)
    so = None if S == 1 else np.linspace(0, M, S + 1).astype(np.int32)
    if S == 1:
        plain = _plain(ft2, x, w, b)
        ref = plain.copy()
        rb, rk, rnf = oracle.bounds(ref, correct_nonfinite=True)
        y, bnd, keys, nf, _ = _derive(ft2, x, w, b, S=1)
        assert np.array_equal(bnd, rb) and np.array_equal(keys, _tp_keys(rk)) and np.array_equal(nf, rnf)
        assert np.array_equal(y, ref)
    else:
        _check_derive(ft2, x, w, b, so, S)


def test_prefill_derive_ragged_sequences_and_padding(ft2):
    # uneven prompt lengths, padding rows before the first and after the last sequence (A18),
    # sequences sharing warps and tiles
    M, N, K = 700, 512, 256
    x, w, b = _operands(M, N, K, seed=41)
    so = np.array([5, 6, 40, 41, 200, 333, 334, 690], np.int32)
    _check_derive(ft2, x, w, b, so, so.size - 1)


def test_prefill_derive_many_sequences_global_path(ft2):
    # more sequences than the per-CTA shared-memory table (512): direct global atomics
    M, N, K = 1400, 256, 128
    x, w, b = _operands(M, N, K, seed=43)
    so = np.arange(0, M + 1, 2, dtype=np.int32)   # 700 sequences of 2 tokens
    _check_derive(ft2, x, w, b, so, so.size - 1)


def test_prefill_derive_nonfinite_corrected(ft2):
    # +Inf / NaN biases make whole columns non-finite: excluded from the bounds (A3/A4),
    # corrected in place (A5/A6), counted per sequence
    M, N, K = 512, 512, 256
    x, w, b = _operands(M, N, K, seed=47)
    b = b.copy()
    b[7] = 0x7F80    # +Inf
    b[300] = 0xFF80  # -Inf
    b[301] = 0x7FC0  # NaN
    so = np.array([0, 100, 256, 512], np.int32)
    rnf = _check_derive(ft2, x, w, b, so, 3)
    assert rnf.sum() == 3 * M


def test_prefill_derive_patch_list_overflow(ft2):
    # more non-finite outputs than the 4096-entry patch list: the last CTA sweeps
    M, N, K = 256, 512, 64
    x, w, b = _operands(M, N, K, seed=53)
    b = b.copy()
    b[0:40] = 0x7FC0
    so = np.array([0, 128, 256], np.int32)
    rnf = _check_derive(ft2, x, w, b, so, 2)
    assert rnf.sum() == 40 * M > 4096


def test_prefill_derive_with_fault_sites(ft2):
    # faults of step 0 (the prefill) land before the derivation (A20): EXP flips can
    # create Inf/NaN that the first-token pass must exclude and correct
    M, N, K = 512, 1024, 256
    x, w, b = _operands(M, N, K, seed=59)
    S = 4
    so = np.linspace(0, M, S + 1).astype(np.int32)
    sites = oracle.make_sites(7, 0, S, oracle.FAULT_EXP, [N] * 3, n_steps=0, prompt_len=M // S)
    for layer in range(3):
        _check_derive(ft2, x, w, b, so, S, sites=sites, layer=layer)


def test_prefill_derive_non_power_of_two_scale(ft2):
    M, N, K = 384, 512, 256
    x, w, b = _operands(M, N, K, seed=61)
    so = np.array([0, 128, 384], np.int32)
    _check_derive(ft2, x, w, b, so, 2, scale=1.25)


def test_prefill_derive_workspace_reuse(ft2):
    # one workspace across calls of different sizes stays consistent
    ws = ft2.make_workspace(64)
    for M, N, K, S in [(512, 512, 128, 4), (1024, 768, 256, 8), (512, 512, 128, 4)]:
        x, w, b = _operands(M, N, K, seed=M + S)
        so = np.linspace(0, M, S + 1).astype(np.int32)
        plain = _plain(ft2, x, w, b)
        rb, _, _ = oracle.bounds(plain.copy(), seq_offsets=so, correct_nonfinite=True)
        _, bnd, _, _, _ = _derive(ft2, x, w, b, so=so, S=S, ws=ws)
        assert np.array_equal(bnd, rb)


# ------------------------------------------------------- split-K (small M) --
# shapes whose units * splits fit one wave (the planner's condition: the splits of a tile wait for each other)
SPLIT_SHAPES = [(256, 8192, 4096), (256, 4096, 11008), (192, 4096, 4096), (512, 2048, 8192), (136, 1032, 4096),
                (512, 4096, 4096)]


@pytest.fixture
def split_on(monkeypatch):
    """The persistent kernel's K split (FT2_PREFILL_SPLITS, read per call;
    -1, the default, lets its planner choose; 0 disables it)."""
    monkeypatch.setenv("FT2_PREFILL_SPLITS", "-1")
    yield


@pytest.mark.parametrize("M,N,K", SPLIT_SHAPES)
def test_split_k_plain_check_and_no_split(ft2, split_on, M, N, K):
    """Grids the tiles cannot fill split K through the fp32 workspace; with
    and without the split the layer is within the GEMM tolerance of the fp64
    oracle, and the CHECK epilogue (same split) is bit-exact vs the oracle's
    R5 on the kernel's own PLAIN output."""
    assert ft2.gemm_workspace_bytes(M, N, K) > 0, "this shape should split"
    x, w, b = _operands(M, N, K, seed=M + K)
    rows = np.unique(np.linspace(0, M - 1, 10).astype(int))
    y_ref, _ = oracle.linear_f64(x[rows], w, b)
    rms = np.sqrt(np.mean(y_ref ** 2, axis=1, keepdims=True))
    tiny = torch.zeros(2, dtype=torch.int64, device="cuda")       # 16 bytes: no split
    outs = []
    for ws in (None, tiny):
        y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=0, workspace=ws)
        torch.cuda.synchronize()
        g = _f64(host(y)[rows])
        assert int((np.abs(g - y_ref) > 1e-2 * np.maximum(np.abs(y_ref), 1e-2 * rms)).sum()) == 0
        outs.append(host(y))
    plain = outs[0]
    S = M
    bnds = np.array([[oracle.f64_to_bf16(-0.2 - 0.001 * i), oracle.f64_to_bf16(0.25)] for i in range(S)], np.uint16)
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    cnt = torch.zeros(S, dtype=torch.int32, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y, bias=dev(b), mode=1, bounds=dev(bnds), num_seqs=S, corrected_count=cnt)
    ref = plain.copy()
    rc = oracle.protect(ref, bnds, row_to_seq=np.arange(M, dtype=np.int32))
    assert np.array_equal(host(y), ref)
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), rc) and rc.sum() > 0
    # the split workspace is self-cleaning: a second call gives the same bits
    y2 = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    ft2.protect_fused_gemm(dev(x), dev(w), y2, bias=dev(b), mode=0)
    assert np.array_equal(host(y2), plain)


@pytest.mark.parametrize("M,N,K,S", [(512, 4096, 4096, 32), (256, 8192, 4096, 16)])
def test_split_k_derive_bit_exact(ft2, split_on, M, N, K, S):
    x, w, b = _operands(M, N, K, seed=S + 3)
    so = np.arange(0, M + 1, M // S).astype(np.int32)
    _check_derive(ft2, x, w, b, so, S)
