"""Statistical fault-injection campaign (config C5 proxy).

One trial = one batch row = one inference with exactly one fault (L88) at a
uniformly drawn (step, linear layer, neuron, bit) site (L90, L95; readings
A11-A13), generated on the GPU by ft2_make_fault_sites and therefore
identical for any sharding of the trial range.  For every batch of trials the
campaign runs, on the same prompts and sites:

  golden_off  fault-free, FT2 off          golden_on  fault-free, FT2 on (fused)
  faulty_off  faults,     FT2 off          faulty_on  faults,     FT2 on (fused)

and counts a *proxy SDC* when a trial's generated tokens differ from the
golden run of the same protection mode.  With random weights greedy decoding
is chaotic (a tiny perturbation flips a token), so a second, magnitude-based
proxy is reported beside it: the relative L2 deviation of the last-position
hidden state (before the final norm) at the faulted step from the golden run,
counted as *large* above 1 (or non-finite) -- the numeric corruption FT2's
range restriction is designed to stop (extreme values and
NaN from exponent flips).  With seeded random weights there is
no semantic notion of a wrong answer, so this proxy is
labelled as such and is never compared with the paper's SDC rates
(parity unpinned).  Reported: proxy-SDC rates with 95% Wald
margins (L282), the reduction 1 - p_on/p_off (L313) and the detection rate
(trials whose row FT2 corrected more neurons in than in its fault-free run).

Sharding: rank r of W takes trials [r*n/W, (r+1)*n/W); per-rank counters are
summed with one all_reduce at the end (the only collective).
"""
from __future__ import annotations

import dataclasses
import math

import torch

from . import ft2 as F2
from .runner import Runner

MODEL_NAMES = {0: "1bit", 1: "2bit", 2: "exp"}


@dataclasses.dataclass
class CampaignResult:
    trials: int = 0
    sdc_off: int = 0
    sdc_on: int = 0
    detected_on: int = 0
    golden_mismatch: int = 0   # fault-free FT2-on vs FT2-off token differences (false-positive proxy)
    fault_free_corrected: int = 0   # rows whose fault-free FT2-on run clipped at least one neuron
    dev_large_off: int = 0     # faulted-step hidden state: relative deviation > 1 or non-finite, FT2 off
    dev_large_on: int = 0      # ... FT2 on
    nonfinite_off: int = 0     # faulted-step hidden state holds NaN / Inf, FT2 off
    nonfinite_on: int = 0      # ... FT2 on

    def add(self, other: "CampaignResult"):
        for f in dataclasses.fields(self):
            setattr(self, f.name, getattr(self, f.name) + getattr(other, f.name))

    def as_tensor(self, device):
        return torch.tensor([getattr(self, f.name) for f in dataclasses.fields(self)], dtype=torch.int64,
                            device=device)

    @classmethod
    def from_tensor(cls, t):
        return cls(*[int(v) for v in t.tolist()])

    def summary(self):
        n = max(1, self.trials)
        p_off, p_on = self.sdc_off / n, self.sdc_on / n
        return {
            "trials": self.trials,
            "proxy_sdc_off": p_off, "proxy_sdc_off_margin95": wald_margin(p_off, n),
            "proxy_sdc_on": p_on, "proxy_sdc_on_margin95": wald_margin(p_on, n),
            "proxy_sdc_reduction": (1.0 - p_on / p_off) if p_off > 0 else None,
            "detection_rate": self.detected_on / n,
            "fault_free_mismatch_rate": self.golden_mismatch / n,
            "fault_free_correction_rate": self.fault_free_corrected / n,
            "large_deviation_off": self.dev_large_off / n,
            "large_deviation_off_margin95": wald_margin(self.dev_large_off / n, n),
            "large_deviation_on": self.dev_large_on / n,
            "large_deviation_on_margin95": wald_margin(self.dev_large_on / n, n),
            "large_deviation_reduction": (1.0 - self.dev_large_on / self.dev_large_off) if self.dev_large_off else None,
            "nonfinite_hidden_off": self.nonfinite_off / n,
            "nonfinite_hidden_on": self.nonfinite_on / n,
            "label": "proxy SDC = generated tokens differ from the golden run (random weights; not the paper's SDC); "
                     "large deviation = faulted-step hidden state off by > 100% (L2) or non-finite",
        }


def wald_margin(p: float, n: int, z: float = 1.96) -> float:
    """95% Wald margin of a proportion."""
    return z * math.sqrt(max(p * (1.0 - p), 0.0) / max(n, 1))


def trial_range(n_trials: int, world: int, rank: int):
    """Contiguous trial shard [begin, end) of `rank`."""
    return (rank * n_trials) // world, ((rank + 1) * n_trials) // world


OFF_MODE = "fused_plain"   # FT2 off = the same tcgen05 GEMM without the check


def golden_runs(runner: Runner, prompt_ids: torch.Tensor, use_graph: bool = True, off_mode: str = OFF_MODE):
    """Fault-free generations with FT2 off and on (the golden runs of every
    batch: prompts and weights are fixed for the whole campaign), plus the
    fault-free corrected-neuron count of every row with FT2 on.

    FT2 off runs the same tcgen05 GEMM as FT2 on, without the check
    ("fused_plain"), so golden_off and golden_on differ only where the
    fault-free check clips (off_mode="off" would compare against cuBLAS,
    whose different summation order alone changes greedy tokens)."""
    runner.set_sites(None)
    g_off = runner.generate(prompt_ids, off_mode, use_graph=use_graph).clone()
    h_off = runner.h_trace.clone()
    g_on = runner.generate(prompt_ids, "fused", use_graph=use_graph).clone()
    h_on = runner.h_trace.clone()
    g_corr = (runner.state.corrected.sum(0) + runner.state.nonfinite.sum(0)).clone()
    return Golden(g_off, g_on, g_corr, h_off, h_on)


@dataclasses.dataclass
class Golden:
    """Fault-free reference runs of one batch of prompts."""
    tok_off: torch.Tensor    # [B, G] generated ids, FT2 off
    tok_on: torch.Tensor     # [B, G] FT2 on
    corr_on: torch.Tensor    # [B] neurons the fault-free FT2-on run corrected
    h_off: torch.Tensor      # [G, B, hidden] last-position hidden state per step
    h_on: torch.Tensor


def site_steps(runner: Runner) -> torch.Tensor:
    """Step field (0 = prefill) of the armed site of every batch row (ft2_fault_site layout)."""
    raw = runner.sites_buf.view(runner.B, F2.SITE_BYTES)
    return (raw[:, 4].long() | (raw[:, 5].long() << 8))


def hidden_deviation(h: torch.Tensor, h_ref: torch.Tensor, steps: torch.Tensor):
    """Per row: relative L2 deviation of the hidden state at its faulted step
    (fp32), and whether that state holds a non-finite value."""
    idx = torch.arange(h.shape[1], device=h.device)
    a = h[steps, idx].float()
    r = h_ref[steps, idx].float()
    nonfin = ~torch.isfinite(a).all(dim=1)
    d = (a - r).norm(dim=1) / r.norm(dim=1).clamp_min(1e-30)
    d = torch.where(nonfin | torch.isnan(d), torch.full_like(d, float("inf")), d)
    return d, nonfin


def run_batch(runner: Runner, prompt_ids: torch.Tensor, seed: int, trial0: int, fault_model: int,
              step_policy: int = 0, golden=None, take: int | None = None, use_graph: bool = True,
              off_mode: str = OFF_MODE) -> CampaignResult:
    """One batch of B trials (rows) on the runner; returns the counters of its
    first `take` rows (default all B).  `golden` = golden_runs(...) of the same
    prompts, computed here when None.  With use_graph the faulty generations
    replay per-step CUDA graphs captured once (the sites live in the runner's
    stable sites_buf, rewritten per batch by ft2_make_fault_sites).

    A trial is *detected* when FT2 corrected more neurons in its row than in
    the fault-free run of the same row (the check also clips a few fault-free
    outliers; those are counted as fault_free_corrected)."""
    B = runner.B
    take = B if take is None else take
    g = golden if golden is not None else golden_runs(runner, prompt_ids, use_graph, off_mode)
    runner.make_sites(seed, trial0, fault_model, step_policy=step_policy)
    steps = site_steps(runner)
    faulty_off = runner.generate(prompt_ids, off_mode, use_graph=use_graph)[:take].clone()
    d_off, nf_off = hidden_deviation(runner.h_trace, g.h_off, steps)
    faulty_on = runner.generate(prompt_ids, "fused", use_graph=use_graph)[:take].clone()
    d_on, nf_on = hidden_deviation(runner.h_trace, g.h_on, steps)
    corrected = (runner.state.corrected.sum(0) + runner.state.nonfinite.sum(0))[:take]   # per trial row
    runner.set_sites(None)
    r = CampaignResult()
    r.trials = take
    r.sdc_off = int((faulty_off != g.tok_off[:take]).any(1).sum().item())
    r.sdc_on = int((faulty_on != g.tok_on[:take]).any(1).sum().item())
    r.detected_on = int((corrected > g.corr_on[:take]).sum().item())
    r.golden_mismatch = int((g.tok_on[:take] != g.tok_off[:take]).any(1).sum().item())
    r.fault_free_corrected = int((g.corr_on[:take] > 0).sum().item())
    r.dev_large_off = int((d_off[:take] > 1.0).sum().item())
    r.dev_large_on = int((d_on[:take] > 1.0).sum().item())
    r.nonfinite_off = int(nf_off[:take].sum().item())
    r.nonfinite_on = int(nf_on[:take].sum().item())
    return r


@dataclasses.dataclass
class PairedResult:
    """Coverage c against the reference coverage (FT2's critical layers) on the
    same trials: the discordant pairs of a McNemar comparison."""
    trials: int = 0
    sdc: int = 0               # proxy SDC under coverage c
    dev_large: int = 0         # large hidden deviation under coverage c
    detected: int = 0
    sdc_only_c: int = 0        # SDC under c but not under the reference
    sdc_only_ref: int = 0      # SDC under the reference but not under c
    dev_only_c: int = 0
    dev_only_ref: int = 0

    def add(self, other: "PairedResult"):
        for f in dataclasses.fields(self):
            setattr(self, f.name, getattr(self, f.name) + getattr(other, f.name))

    def as_tensor(self, device):
        return torch.tensor([getattr(self, f.name) for f in dataclasses.fields(self)], dtype=torch.int64,
                            device=device)

    @classmethod
    def from_tensor(cls, t):
        return cls(*[int(v) for v in t.tolist()])

    def summary(self):
        n = max(1, self.trials)
        p, q = self.sdc / n, self.dev_large / n
        return {"trials": self.trials, "proxy_sdc": p, "proxy_sdc_margin95": wald_margin(p, n),
                "large_deviation": q, "large_deviation_margin95": wald_margin(q, n),
                "detection_rate": self.detected / n,
                "vs_ft2_discordant": {"sdc_only_this": self.sdc_only_c, "sdc_only_ft2": self.sdc_only_ref,
                                      "large_dev_only_this": self.dev_only_c, "large_dev_only_ft2": self.dev_only_ref}}


def run_coverages(runners: dict, off_runner: Runner, prompt_ids: torch.Tensor, seed: int, trial0: int,
                  fault_model: int, goldens: dict, take: int | None = None, ref: str = "ft2",
                  use_graph: bool = True, off_mode: str = OFF_MODE) -> dict:
    """One batch of trials under several protection coverages (Table 1,
    L164-L177: "ft2", "maximals", "globalclipper", "all", "none" = Ranger's
    linear-layer coverage; or caller-supplied-bounds runners) on IDENTICAL
    sites: the sites are generated once into the shared site buffer, the
    unprotected run is shared, and every coverage runner (Runner.with_coverage
    of off_runner, same weights) replays its protected generation.  goldens:
    coverage -> golden_runs of that runner ("off" -> the unprotected golden).
    Returns coverage -> PairedResult (discordance against `ref`)."""
    B = off_runner.B
    take = B if take is None else take
    off_runner.make_sites(seed, trial0, fault_model)
    steps = site_steps(off_runner)
    g_off = goldens["off"]
    faulty_off = off_runner.generate(prompt_ids, off_mode, use_graph=use_graph)[:take].clone()
    d_off, _ = hidden_deviation(off_runner.h_trace, g_off.h_off, steps)
    sdc, dev, det = {}, {}, {}
    for cov, r_ in runners.items():
        r_.sites = r_.sites_buf   # same buffer (shared): arm the sites on this runner too
        out = r_.generate(prompt_ids, "fused", use_graph=use_graph)[:take]
        g = goldens[cov]
        sdc[cov] = (out != g.tok_on[:take]).any(1)
        d, _ = hidden_deviation(r_.h_trace, g.h_on, steps)
        dev[cov] = d[:take] > 1.0
        corr = (r_.state.corrected.sum(0) + r_.state.nonfinite.sum(0))[:take]
        det[cov] = corr > g.corr_on[:take]
        r_.sites = None
    off_runner.set_sites(None)
    sdc["off"] = (faulty_off != g_off.tok_off[:take]).any(1)
    dev["off"] = d_off[:take] > 1.0
    det["off"] = torch.zeros_like(sdc["off"])
    res = {}
    for cov in list(runners) + ["off"]:
        p = PairedResult(trials=take, sdc=int(sdc[cov].sum()), dev_large=int(dev[cov].sum()),
                         detected=int(det[cov].sum()))
        if ref in sdc:
            p.sdc_only_c = int((sdc[cov] & ~sdc[ref]).sum())
            p.sdc_only_ref = int((sdc[ref] & ~sdc[cov]).sum())
            p.dev_only_c = int((dev[cov] & ~dev[ref]).sum())
            p.dev_only_ref = int((dev[ref] & ~dev[cov]).sum())
        res[cov] = p
    return res


def campaign_prompts(runner: Runner, prompt_seed: int = 7) -> torch.Tensor:
    gen = torch.Generator().manual_seed(prompt_seed)
    return torch.randint(0, runner.cfg.vocab, (runner.B, runner.T), generator=gen).to(runner.device)


def run_campaign(runner: Runner, n_trials: int, seed: int, fault_model: int, rank: int = 0, world: int = 1,
                 group=None, prompt_seed: int = 7, use_graph: bool = True) -> CampaignResult:
    """This rank's share of n_trials (batches of runner.B rows), counters summed over ranks."""
    t0, t1 = trial_range(n_trials, world, rank)
    total = CampaignResult()
    prompts = campaign_prompts(runner, prompt_seed)
    golden = golden_runs(runner, prompts, use_graph)
    t = t0
    while t < t1:
        total.add(run_batch(runner, prompts, seed, t, fault_model, golden=golden, take=min(runner.B, t1 - t),
                            use_graph=use_graph))
        t += runner.B
    if world > 1:
        import torch.distributed as dist
        v = total.as_tensor(runner.device)
        dist.all_reduce(v, group=group)
        total = CampaignResult.from_tensor(v)
    return total
