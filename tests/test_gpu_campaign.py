"""Fault-injection campaign on a tiny synthetic model (GPU): determinism of the
golden runs, sites bit-exact with the oracle, injected faults actually reach
the outputs, and shard sums equal the unsharded campaign."""
import numpy as np
import pytest
import torch

import oracle
import oracle.stats  # noqa: F401  (submodule used below)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tiny():
    from paper_conf_hpdc_sunzmg00y25_b200.runner import ModelConfig, Runner
    cfg = ModelConfig("llama", 256, 512, 2, 4, 512, 512, False)
    return Runner(cfg, batch=16, prompt_len=8, gen_len=6, seed=3)


def test_campaign_sites_match_oracle(tiny):
    from paper_conf_hpdc_sunzmg00y25_b200 import ft2
    w = tiny.cfg.linear_widths()
    for model in (0, 1, 2):
        s = ft2.make_fault_sites(11, 100, 16, model, w, n_steps=5, prompt_len=8)
        ref = oracle.make_sites(11, 100, 16, model, w, 5, 8)
        assert s.cpu().numpy().tobytes() == ref.tobytes()


def test_golden_runs_are_deterministic(tiny):
    p = torch.randint(0, 512, (16, 8), generator=torch.Generator().manual_seed(1)).cuda()
    a = tiny.generate(p, "fused", use_graph=False).clone()
    b = tiny.generate(p, "fused", use_graph=False).clone()
    c = tiny.generate(p, "fused", use_graph=True).clone()
    assert torch.equal(a, b) and torch.equal(a, c)


def test_exponent_faults_reach_outputs_and_ft2_detects(tiny):
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    p = torch.randint(0, 512, (16, 8), generator=torch.Generator().manual_seed(2)).cuda()
    tot = campaign.CampaignResult()
    for t0 in range(0, 64, 16):
        tot.add(campaign.run_batch(tiny, p, seed=5, trial0=t0, fault_model=2))
    s = tot.summary()
    assert tot.trials == 64
    assert 0 <= tot.sdc_on <= tot.trials and 0 <= tot.sdc_off <= tot.trials
    assert tot.detected_on > 0          # EXP flips in critical layers are corrected by FT2
    assert s["proxy_sdc_off_margin95"] == pytest.approx(oracle.stats.wald_margin(tot.sdc_off / 64, 64))


def test_shards_sum_to_unsharded(tiny):
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    full = campaign.run_campaign(tiny, 32, seed=9, fault_model=0)
    parts = campaign.CampaignResult()
    gen = torch.Generator().manual_seed(7)
    prompts = torch.randint(0, tiny.cfg.vocab, (tiny.B, tiny.T), generator=gen).cuda()
    for r in range(2):      # rank r of 2 runs its trial range; counters add up
        b, e = campaign.trial_range(32, 2, r)
        for t in range(b, e, tiny.B):
            parts.add(campaign.run_batch(tiny, prompts, 9, t, 0))
    assert parts == full


def test_coverage_none_equals_unprotected_and_all_detects():
    """Table 1 coverages: with no protected linear layer (Ranger's linear-layer
    coverage) FT2-on is FT2-off, trial by trial; covering every linear layer
    corrects at least one fault."""
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    from paper_conf_hpdc_sunzmg00y25_b200.runner import ModelConfig, Runner
    cfg = ModelConfig("llama", 256, 512, 2, 4, 512, 512, False)
    p = torch.randint(0, 512, (16, 8), generator=torch.Generator().manual_seed(4)).cuda()
    none = Runner(cfg, batch=16, prompt_len=8, gen_len=6, seed=3, coverage="none")
    r = campaign.run_batch(none, p, seed=5, trial0=0, fault_model=2)
    assert none.n_crit == 0 and r.sdc_on == r.sdc_off and r.detected_on == 0 and r.golden_mismatch == 0
    full = Runner(cfg, batch=16, prompt_len=8, gen_len=6, seed=3, coverage="all")
    assert full.n_crit == 7 * 2
    r = campaign.run_batch(full, p, seed=5, trial0=0, fault_model=2)
    assert r.detected_on > 0


def test_nan_vulnerable_profile_matches_oracle(tiny):
    """PAPER.md L202 / Fig. 8(b): NaN-vulnerable share of each linear layer's
    fault-free output; block 0's q_proj counts are recomputed with the oracle
    from the same (deterministic) cuBLAS output."""
    import torch.nn.functional as F
    p = torch.randint(0, 512, (16, 8), generator=torch.Generator().manual_seed(6)).cuda()
    share, counts, elems = tiny.profile_nan_vulnerable(p)
    assert set(share) == set(tiny.lin_names) and all(0.0 <= v <= 1.0 for v in share.values())
    assert counts.shape == (2, len(tiny.lin_names), 16)
    blk = tiny.blocks[0]
    pos = torch.arange(8, device="cuda")
    x = tiny._embed(p, pos.unsqueeze(0).expand(16, 8))
    h2 = tiny._norm(x, blk.ln1_w, blk.ln1_b).reshape(-1, tiny.cfg.hidden)
    y = F.linear(h2, blk.w["q_proj"], blk.b["q_proj"])
    yh = y.view(torch.int16).cpu().numpy().view(np.uint16)
    want = oracle.nan_vulnerable_count(yh, seq_offsets=np.arange(0, 17 * 8, 8))
    assert counts[0, 0].numpy().astype(np.uint32).tolist() == want.tolist()
    assert int(elems[0]) == 8 * tiny.cfg.hidden


def test_graphed_faulty_runs_equal_eager(tiny):
    """Per-step CUDA graphs of the faulty generations (captured once, sites
    rewritten in place per batch) give the same tokens and the same FT2
    counters as eager decode, batch after batch."""
    p = torch.randint(0, 512, (16, 8), generator=torch.Generator().manual_seed(8)).cuda()
    for trial0 in (0, 16, 32):
        for mode in ("off", "fused"):
            tiny.make_sites(5, trial0, 2)
            e = tiny.generate(p, mode, use_graph=False).clone()
            ec = (tiny.state.corrected.clone(), tiny.state.nonfinite.clone())
            tiny.make_sites(5, trial0, 2)
            g = tiny.generate(p, mode, use_graph=True).clone()
            assert torch.equal(e, g), (trial0, mode)
            assert torch.equal(ec[0], tiny.state.corrected) and torch.equal(ec[1], tiny.state.nonfinite)
    tiny.set_sites(None)


def test_partial_batch_counts_only_its_rows(tiny):
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    prompts = campaign.campaign_prompts(tiny)
    gold = campaign.golden_runs(tiny, prompts)
    full = campaign.run_batch(tiny, prompts, 3, 0, 2, golden=gold)
    part = campaign.run_batch(tiny, prompts, 3, 0, 2, golden=gold, take=5)
    assert part.trials == 5 and full.trials == 16
    assert part.sdc_off <= full.sdc_off and part.detected_on <= full.detected_on
    eager = campaign.run_batch(tiny, prompts, 3, 0, 2, golden=gold, use_graph=False)
    assert eager == full
