"""ft2_host_norm (the runner's host-model LayerNorm / RMSNorm; include/ft2.h)
against plain PyTorch fp32 norms of the same 16-bit inputs.  Not part of the
FT2 method, so no oracle: the reference is the textbook formula in fp32,
rounded once to the output dtype (tolerance: 2 ulps of bf16 / fp16)."""
import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ft2():
    import paper_conf_hpdc_sunzmg00y25_b200 as m
    return m


def _ref(x, w, b, eps, rms):
    xf, wf = x.float(), w.float()
    if rms:
        y = xf * torch.rsqrt(xf.pow(2).mean(-1, keepdim=True) + eps) * wf
    else:
        m = xf.mean(-1, keepdim=True)
        y = (xf - m) * torch.rsqrt((xf - m).pow(2).mean(-1, keepdim=True) + eps) * wf
        if b is not None:
            y = y + b.float()
    return y.to(x.dtype)


@pytest.mark.parametrize("rows,n", [(1, 8), (32, 768), (33, 2048), (7, 4096), (32, 5120), (3, 8192), (129, 1000 // 8 * 8)])
@pytest.mark.parametrize("rms", [False, True])
@pytest.mark.parametrize("dtype", [torch.bfloat16, torch.float16])
def test_host_norm_matches_fp32_reference(ft2, rows, n, rms, dtype):
    g = torch.Generator(device="cuda").manual_seed(rows * 131 + n)
    x = (torch.randn(rows, n, device="cuda", generator=g) * 3 + 0.5).to(dtype)
    w = (torch.rand(n, device="cuda", generator=g) + 0.5).to(dtype)
    b = None if rms else (torch.randn(n, device="cuda", generator=g) * 0.1).to(dtype)
    y = torch.empty_like(x)
    ft2.host_norm(x, w, y, bias=b, eps=1e-5, rms=rms)
    torch.cuda.synchronize()
    ref = _ref(x, w, b, 1e-5, rms)
    ulp = 2.0 ** -7 if dtype == torch.bfloat16 else 2.0 ** -10
    torch.testing.assert_close(y.float(), ref.float(), rtol=2 * ulp, atol=2 * ulp)


def test_host_norm_strided_rows_and_torch_layer_norm(ft2):
    base = torch.randn(32, 2048 + 64, device="cuda").to(torch.bfloat16)
    x = base[:, :2048]
    w = torch.rand(2048, device="cuda").to(torch.bfloat16) + 0.5
    b = torch.randn(2048, device="cuda").to(torch.bfloat16)
    out = torch.zeros(32, 2048 + 128, device="cuda", dtype=torch.bfloat16)
    y = out[:, :2048]
    ft2.host_norm(x, w, y, bias=b, eps=1e-5)
    torch.cuda.synchronize()
    assert torch.all(out[:, 2048:] == 0)                      # nothing written past n
    t = torch.nn.functional.layer_norm(x, (2048,), w, b, 1e-5)
    torch.testing.assert_close(y.float(), t.float(), rtol=2 ** -6, atol=2 ** -6)


def test_host_norm_errors(ft2):
    from paper_conf_hpdc_sunzmg00y25_b200._lib import FT2Error
    x = torch.randn(4, 8200, device="cuda").to(torch.bfloat16)
    with pytest.raises(FT2Error, match="UNSUPPORTED"):
        ft2.host_norm(x, x[0], torch.empty_like(x))            # n > 8192
    x = torch.randn(4, 12, device="cuda").to(torch.bfloat16)
    with pytest.raises(FT2Error, match="UNSUPPORTED"):
        ft2.host_norm(x, x[0], torch.empty_like(x))            # n % 8 != 0
    x = torch.randn(4, 16, device="cuda")
    with pytest.raises(FT2Error, match="UNSUPPORTED"):
        ft2.host_norm(x, x[0], torch.empty_like(x))            # fp32
    x = torch.randn(4, 16, device="cuda").to(torch.bfloat16)
    with pytest.raises(FT2Error, match="INVALID_ARG"):
        ft2.host_norm(x, x[0], torch.empty_like(x), eps=-1.0)
    e = torch.empty(0, 16, device="cuda", dtype=torch.bfloat16)
    ft2.host_norm(e, x[0], torch.empty_like(e))                # rows == 0: no launch


@pytest.mark.parametrize("rows,n", [(1, 8), (32, 8192), (33, 11008), (4096, 2048)])
@pytest.mark.parametrize("dtype", [torch.bfloat16, torch.float16])
def test_host_act_relu_bit_exact(ft2, rows, n, dtype):
    g = torch.Generator(device="cuda").manual_seed(rows + n)
    a = torch.randn(rows, n, device="cuda", generator=g).to(dtype)
    a.view(-1)[::997] = float("nan")
    a.view(-1)[5::1009] = float("-inf")
    y = torch.empty_like(a)
    ft2.host_act(a, y)
    torch.cuda.synchronize()
    ref = torch.relu(a)
    assert torch.equal(torch.isnan(y), torch.isnan(ref))      # NaN propagates, as torch.relu
    m = ~torch.isnan(ref)
    assert torch.equal(y[m], ref[m])
    assert not torch.any(y[m].view(torch.int16) < 0)           # no negative (or -0) outputs


@pytest.mark.parametrize("rows,n", [(1, 8), (32, 11008), (7, 13824)])
@pytest.mark.parametrize("dtype", [torch.bfloat16, torch.float16])
def test_host_act_silu_mul_matches_torch(ft2, rows, n, dtype):
    g = torch.Generator(device="cuda").manual_seed(rows * 7 + n)
    gu = (torch.randn(rows, 2 * n, device="cuda", generator=g) * 4).to(dtype)
    a, b = gu[:, :n], gu[:, n:]                                  # strided views, as the fused gate_up GEMM gives
    y = torch.empty(rows, n, device="cuda", dtype=dtype)
    ft2.host_act(a, y, b=b, act="silu_mul")
    torch.cuda.synchronize()
    ref = torch.nn.functional.silu(a) * b
    ulp = 2.0 ** -7 if dtype == torch.bfloat16 else 2.0 ** -10
    torch.testing.assert_close(y.float(), ref.float(), rtol=2 * ulp, atol=1e-3)
    # the fp32 formula rounded twice, as torch does: almost all bit-identical
    assert (y != ref).float().mean().item() < 1e-3


def test_host_act_errors(ft2):
    from paper_conf_hpdc_sunzmg00y25_b200._lib import FT2Error
    a = torch.randn(4, 16, device="cuda").to(torch.bfloat16)
    from paper_conf_hpdc_sunzmg00y25_b200._lib import check, load
    with pytest.raises(FT2Error, match="INVALID_ARG"):   # silu_mul with b NULL
        check("ft2_host_act", load().ft2_host_act(a.data_ptr(), 16, None, 0, a.data_ptr(), 16, 4, 16, 1, 0, None))
    with pytest.raises(FT2Error, match="MISALIGNED"):
        x = torch.randn(4, 12, device="cuda").to(torch.bfloat16)
        ft2.host_act(x, torch.empty_like(x))
    e = torch.empty(0, 16, device="cuda", dtype=torch.bfloat16)
    ft2.host_act(e, torch.empty_like(e))


def test_pdl_chain_graph_replay():
    """the early-trigger chain host_norm -> fused GEMM -> host_act
    -> fused GEMM, captured once and replayed with new inputs each time, must
    give bit-identical outputs with programmatic dependent launch on
    (FT2_GEMM_PDL=1, the default) and off (plain stream order), and with the
    host-model kernels replaced by torch's (FT2_HOST_NORM=0 equivalent: the
    same chain with torch ops feeding the GEMMs, compared against eager
    launches).  Each variant runs in its own process (the knobs are read
    once)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = r'''
import sys, torch, hashlib
sys.path.insert(0, ROOT)
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
import ft2_synth
H, F, B = 2048, 8192, 32
w1 = ft2_synth.gen_bf16_torch((F, H), 1, 3, scale_log2=-6, device="cuda")
w2 = ft2_synth.gen_bf16_torch((H, F), 2, 3, scale_log2=-7, device="cuda")
lnw = torch.ones(H, dtype=torch.bfloat16, device="cuda"); lnb = torch.zeros(H, dtype=torch.bfloat16, device="cuda")
bnd = torch.tensor([[-0.25, 0.25]], dtype=torch.bfloat16, device="cuda")
x = torch.empty((B, H), dtype=torch.bfloat16, device="cuda")
h = torch.empty_like(x); f = torch.empty((B, F), dtype=torch.bfloat16, device="cuda")
a = torch.empty_like(f); y = torch.empty((B, H), dtype=torch.bfloat16, device="cuda")
cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
host = HOST
def chain():
    if host:
        ft2.host_norm(x, lnw, h, bias=lnb, eps=1e-5)
    else:
        h.copy_(torch.nn.functional.layer_norm(x, (H,), lnw, lnb, 1e-5))
    ft2.protect_fused_gemm(h, w1, f, mode=0 | 16)
    if host:
        ft2.host_act(f, a)
    else:
        a.copy_(torch.relu(f))
    ft2.protect_fused_gemm(a, w2, y, mode=1 | 16, bounds=bnd, num_seqs=1, corrected_count=cnt)
def fill(i):
    x.copy_(ft2_synth.gen_bf16_torch((B, H), 100 + i, 3, device="cuda"))
fill(0); chain(); torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    chain()
dig = hashlib.sha256()
for i in range(6):
    fill(i); cnt.zero_(); g.replay(); torch.cuda.synchronize()
    got = (y.clone(), int(cnt.item()))
    fill(i); cnt.zero_(); chain(); torch.cuda.synchronize()    # eager, stream order
    assert torch.equal(got[0].view(torch.int16), y.view(torch.int16)) and got[1] == int(cnt.item()), i
    dig.update(y.view(torch.int16).cpu().numpy().tobytes())
print("digest", dig.hexdigest())
'''.replace("ROOT", repr(root))
    digests = {}
    for host in (1, 0):
        for pdl in ("1", "0"):
            r = subprocess.run([sys.executable, "-c", code.replace("HOST", str(host))],
                               env={**os.environ, "FT2_GEMM_PDL": pdl}, capture_output=True, text=True, timeout=600)
            assert r.returncode == 0, r.stderr[-3000:]
            digests[(host, pdl)] = r.stdout.split("digest")[-1].strip()
    # PDL on/off: identical bits (host kernels and torch kernels alike)
    assert digests[(1, "1")] == digests[(1, "0")]
    assert digests[(0, "1")] == digests[(0, "0")]
