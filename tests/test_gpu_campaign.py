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


def test_paired_coverages_on_identical_sites(tiny):
    """NEXT(4): Table 1 coverages compared on the SAME
    sites -- the unprotected run is shared, every coverage replays its own
    protected generation over shared weights.  "none" (Ranger's linear-layer
    coverage) must equal the unprotected run trial by trial; "ft2" must equal
    the plain campaign path's FT2-on result."""
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    prompts = campaign.campaign_prompts(tiny)
    covs = {c: tiny.with_coverage(c) for c in ("ft2", "maximals", "globalclipper", "all", "none")}
    assert covs["all"].blocks is tiny.blocks and covs["all"].sites_buf is tiny.sites_buf
    assert [covs[c].n_crit for c in covs] == [4 * 2, 2 * 2, 2 * 2, 7 * 2, 0]   # Llama: maximals o/down, gc v/o
    goldens = {c: campaign.golden_runs(r, prompts) for c, r in covs.items()}
    goldens["off"] = campaign.golden_runs(tiny, prompts)
    res = campaign.PairedResult
    tot = {c: res() for c in list(covs) + ["off"]}
    plain = campaign.CampaignResult()
    for t0 in (0, 16, 32):
        r = campaign.run_coverages(covs, tiny, prompts, 5, t0, 2, goldens)
        for c, v in r.items():
            tot[c].add(v)
        plain.add(campaign.run_batch(covs["ft2"], prompts, 5, t0, 2, golden=goldens["ft2"]))
    assert tot["none"].sdc == tot["off"].sdc and tot["none"].detected == 0
    assert tot["ft2"].sdc == plain.sdc_on and tot["ft2"].detected == plain.detected_on
    assert tot["ft2"].sdc_only_c == 0 and tot["ft2"].sdc_only_ref == 0
    for c, v in tot.items():
        assert v.trials == 48
        # discordant pairs reconstruct the difference of the marginals
        assert v.sdc - tot["ft2"].sdc == v.sdc_only_c - v.sdc_only_ref
        assert v.dev_large - tot["ft2"].dev_large == v.dev_only_c - v.dev_only_ref
    assert tot["all"].detected >= tot["ft2"].detected > 0


def test_supplied_bounds_bypass_the_sweep_and_clip_like_the_oracle(tiny):
    """Caller-supplied (offline) bounds: the first-token sweep is skipped (the
    state holds exactly the supplied bounds, no prefill non-finite count),
    every-token checks use them (R5, bit-exact on the layer's own PLAIN
    output), and bounds wide enough to clip nothing reproduce the unprotected
    generation exactly."""
    import torch.nn.functional as F
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    prompts = campaign.campaign_prompts(tiny)
    ref_plain = tiny.generate(prompts, "fused_plain").clone()
    wide = torch.tensor([-3.0e38, 3.0e38], dtype=torch.bfloat16).expand(tiny.n_crit, 2)
    tiny.set_supplied_bounds(wide)
    try:
        out = tiny.generate(prompts, "fused").clone()
        assert torch.equal(out, ref_plain)
        assert int(tiny.state.corrected.sum()) == 0 and int(tiny.state.nonfinite.sum()) == 0
        narrow = torch.tensor([-0.05, 0.05], dtype=torch.bfloat16).expand(tiny.n_crit, 2)
        tiny.set_supplied_bounds(narrow)
        tiny.generate(prompts, "fused")
        st = tiny.state
        assert torch.equal(st.bounds, narrow.unsqueeze(1).expand(tiny.n_crit, tiny.B, 2).to(st.bounds.device))
        assert int(st.corrected.sum()) > 0 and int(st.nonfinite.sum()) == 0
        # one decode layer call against the oracle: CHECK == R5(PLAIN) with the supplied bounds
        blk = tiny.blocks[1]
        x2 = torch.randn(tiny.B, tiny.cfg.hidden, device="cuda").to(torch.bfloat16)
        tiny.mode = "fused_plain"
        plain = tiny._linear(x2, blk, "v_proj", "decode").clone()
        tiny.mode = "fused"
        chk = tiny._linear(x2, blk, "v_proj", "decode").clone()
        ref = plain.view(torch.int16).cpu().numpy().view(np.uint16).copy()
        b = narrow[0].view(torch.int16).numpy().view(np.uint16).reshape(1, 2)
        oracle.protect(ref, b)
        assert np.array_equal(chk.view(torch.int16).cpu().numpy().view(np.uint16), ref)
        # the prefill outputs are checked too: block 0's v_proj output lies within the bounds
        tiny.set_supplied_bounds(narrow)
        pos = torch.arange(tiny.T, device="cuda")
        x = tiny._embed(prompts, pos.unsqueeze(0).expand(tiny.B, tiny.T))
        h2 = tiny._norm(x, tiny.blocks[0].ln1_w, tiny.blocks[0].ln1_b).reshape(-1, tiny.cfg.hidden)
        y = tiny._linear(h2, tiny.blocks[0], "v_proj", "prefill").float()
        lo, hi = float(narrow[0, 0]), float(narrow[0, 1])
        assert float(y.max()) <= hi and float(y.min()) >= lo
        yr = F.linear(h2, tiny.blocks[0].w["v_proj"]).float()
        assert float(yr.max()) > hi                # so the check really clipped
    finally:
        tiny.set_supplied_bounds(None)


def test_offline_profiled_bounds_match_oracle(tiny):
    """profile_offline_bounds: per protected layer, min / max over every output
    of every profiling batch (x2), equal to the oracle's bounds of the
    concatenated outputs (block 0's v_proj recomputed with the same cuBLAS call)."""
    import torch.nn.functional as F
    gens = [torch.Generator().manual_seed(40 + i) for i in range(2)]
    batches = [torch.randint(0, 512, (16, 8), generator=g).cuda() for g in gens]
    b = tiny.profile_offline_bounds(batches)
    assert b.shape == (tiny.n_crit, 2)
    ys = []
    pos = torch.arange(8, device="cuda")
    for p in batches:
        x = tiny._embed(p, pos.unsqueeze(0).expand(16, 8))
        h2 = tiny._norm(x, tiny.blocks[0].ln1_w, tiny.blocks[0].ln1_b).reshape(-1, tiny.cfg.hidden)
        ys.append(F.linear(h2, tiny.blocks[0].w["v_proj"]).view(torch.int16).cpu().numpy().view(np.uint16))
    want, _, _ = oracle.bounds(np.ascontiguousarray(np.concatenate(ys)), scale=2.0)
    cid = tiny._crit_id(0, "v_proj")
    assert b[cid].view(torch.int16).cpu().numpy().view(np.uint16).tolist() == want.reshape(-1).tolist()


def test_hidden_deviation_proxy(tiny):
    from paper_conf_hpdc_sunzmg00y25_b200 import campaign
    prompts = campaign.campaign_prompts(tiny)
    gold = campaign.golden_runs(tiny, prompts)
    tot = campaign.CampaignResult()
    for t0 in range(0, 64, 16):
        tot.add(campaign.run_batch(tiny, prompts, 5, t0, 2, golden=gold))
    assert 0 <= tot.dev_large_on <= tot.trials and 0 <= tot.dev_large_off <= tot.trials
    assert tot.nonfinite_off <= tot.dev_large_off and tot.nonfinite_on <= tot.dev_large_on
    # fault-free: zero deviation against itself
    steps = torch.zeros(tiny.B, dtype=torch.long, device="cuda")
    d, nf = campaign.hidden_deviation(gold.h_on, gold.h_on, steps)
    assert float(d.max()) == 0.0 and not bool(nf.any())
