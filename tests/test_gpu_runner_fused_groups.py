"""Runner with horizontally fused projections (q/k/v, Llama gate/up): the
protected layer (v_proj, up_proj) is a column slice of one GEMM.  Its
first-token bounds must be the oracle's R2-R4 on exactly that slice of the
group's output, its decode check must touch only that slice, and graph and
eager generation must agree."""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle
from gpu_util import host

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", params=["opt", "llama"])
def fused_runner(request):
    from paper_conf_hpdc_sunzmg00y25_b200.runner import ModelConfig, Runner
    if request.param == "opt":
        cfg = ModelConfig("opt", 256, 512, 2, 4, 512, 512, True)
    else:
        cfg = ModelConfig("llama", 256, 512, 2, 4, 512, 512, False)
    return Runner(cfg, batch=8, prompt_len=8, gen_len=6, seed=5, fuse_proj=True)


def _prompts(r, seed):
    return torch.randint(0, r.cfg.vocab, (r.B, r.T), generator=torch.Generator().manual_seed(seed)).cuda()


def test_graph_equals_eager_fused_groups(fused_runner):
    r = fused_runner
    p = _prompts(r, 1)
    for mode in ("off", "fused", "standalone"):
        a = r.generate(p, mode, use_graph=False).clone()
        b = r.generate(p, mode, use_graph=True).clone()
        assert torch.equal(a, b), mode


def test_slice_bounds_are_the_oracle_on_the_group_output(fused_runner):
    """Block 0's protected slice: bounds from the runner's prefill equal the
    oracle's R2-R4 on the same cuBLAS group output (deterministic)."""
    r = fused_runner
    p = _prompts(r, 2)
    r.generate(p, "fused", use_graph=False)
    torch.cuda.synchronize()
    blk = r.blocks[0]
    pos = torch.arange(r.T, device="cuda")
    x = r._embed(p, pos.unsqueeze(0).expand(r.B, r.T))
    h2 = r._norm(x, blk.ln1_w, blk.ln1_b).reshape(-1, r.cfg.hidden)
    y = F.linear(h2, blk.wf["qkv"], blk.bf["qkv"])
    hdim = r.cfg.hidden
    v = np.ascontiguousarray(host(y)[:, 2 * hdim:3 * hdim])
    so = np.arange(0, (r.B + 1) * r.T, r.T).astype(np.int32)
    want, _, _ = oracle.bounds(v, seq_offsets=so, correct_nonfinite=True)
    cid = r._crit_id(0, "v_proj")
    assert np.array_equal(host(r.state.bounds[cid]), want)


def test_fused_check_touches_only_the_protected_slice(fused_runner):
    """Decode-shaped group GEMM in CHECK mode with bounds that clip almost
    everything: the protected slice equals the oracle's R5 on the PLAIN
    output, every other column is the PLAIN output unchanged."""
    import paper_conf_hpdc_sunzmg00y25_b200 as ft2
    r = fused_runner
    blk = r.blocks[1]
    g = "qkv"
    w, b = blk.wf[g], blk.bf[g]
    M = r.B
    x = torch.randn((M, w.shape[1]), device="cuda").to(torch.bfloat16)
    y0 = torch.empty((M, w.shape[0]), dtype=torch.bfloat16, device="cuda")
    ft2.protect_fused_gemm(x, w, y0, bias=b, mode=0)
    c0, c1 = 2 * r.cfg.hidden, 3 * r.cfg.hidden
    bnd = torch.tensor([[-0.05, 0.05]], dtype=torch.bfloat16, device="cuda").repeat(M, 1)
    cnt = torch.zeros(M, dtype=torch.int32, device="cuda")
    y1 = torch.empty_like(y0)
    ft2.protect_fused_gemm(x, w, y1, bias=b, mode=1, col_begin=c0, col_end=c1, bounds=bnd, num_seqs=M,
                           corrected_count=cnt)
    plain, got = host(y0), host(y1)
    ref = np.ascontiguousarray(plain[:, c0:c1])
    rc = oracle.protect(ref, host(bnd), row_to_seq=np.arange(M, dtype=np.int32))
    assert np.array_equal(got[:, c0:c1], ref) and int(rc.sum()) > 0
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), rc)
    assert np.array_equal(got[:, :c0], plain[:, :c0]) and np.array_equal(got[:, c1:], plain[:, c1:])


def test_fault_sites_need_unfused_runner(fused_runner):
    r = fused_runner
    r.make_sites(1, 0, 0)
    try:
        with pytest.raises(ValueError, match="fuse_proj=False"):
            r.generate(_prompts(r, 3), "fused", use_graph=False)
    finally:
        r.set_sites(None)
