"""Fault-injection campaign on a tiny synthetic model (GPU): determinism of the
golden runs, sites bit-exact with the oracle, injected faults actually reach
the outputs, and shard sums equal the unsharded campaign."""
import numpy as np
import pytest
import torch

import oracle

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
