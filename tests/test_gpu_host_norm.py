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
