"""Statistical fault-injection campaign (config C5 proxy).

One trial = one batch row = one inference with exactly one fault (L88) at a
uniformly drawn (step, linear layer, neuron, bit) site (L90, L95; readings
A11-A13), generated on the GPU by ft2_make_fault_sites and therefore
identical for any sharding of the trial range.  For every batch of trials the
campaign runs, on the same prompts and sites:

  golden_off  fault-free, FT2 off          golden_on  fault-free, FT2 on (fused)
  faulty_off  faults,     FT2 off          faulty_on  faults,     FT2 on (fused)

and counts a *proxy SDC* when a trial's generated tokens differ from the
golden run of the same protection mode.  With seeded random weights there is
no semantic notion of a wrong answer, so this proxy is
labelled as such and is never compared with the paper's SDC rates
(parity unpinned).  Reported: proxy-SDC rates with 95% Wald
margins (L282), the reduction 1 - p_on/p_off (L313) and the detection rate
(trials whose FT2 corrected-neuron count is non-zero).

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
            "label": "proxy SDC = generated tokens differ from the golden run (random weights; not the paper's SDC)",
        }


def wald_margin(p: float, n: int, z: float = 1.96) -> float:
    """95% Wald margin of a proportion."""
    return z * math.sqrt(max(p * (1.0 - p), 0.0) / max(n, 1))


def trial_range(n_trials: int, world: int, rank: int):
    """Contiguous trial shard [begin, end) of `rank`."""
    return (rank * n_trials) // world, ((rank + 1) * n_trials) // world


def run_batch(runner: Runner, prompt_ids: torch.Tensor, seed: int, trial0: int, fault_model: int,
              step_policy: int = 0) -> CampaignResult:
    """One batch of B trials (rows) on the runner; returns the counters."""
    B, G = runner.B, runner.G
    widths = runner.cfg.linear_widths()
    sites = F2.make_fault_sites(seed, trial0, B, fault_model, widths, n_steps=G - 1, prompt_len=runner.T,
                                step_policy=step_policy, device=prompt_ids.device)
    runner.sites = None
    golden_off = runner.generate(prompt_ids, "off", use_graph=False).clone()
    golden_on = runner.generate(prompt_ids, "fused", use_graph=False).clone()
    runner.sites = sites
    faulty_off = runner.generate(prompt_ids, "off", use_graph=False).clone()
    faulty_on = runner.generate(prompt_ids, "fused", use_graph=False).clone()
    corrected = runner.state.corrected.sum(0) + runner.state.nonfinite.sum(0)   # per trial row
    runner.sites = None
    r = CampaignResult()
    r.trials = B
    r.sdc_off = int((faulty_off != golden_off).any(1).sum().item())
    r.sdc_on = int((faulty_on != golden_on).any(1).sum().item())
    r.detected_on = int((corrected > 0).sum().item())
    r.golden_mismatch = int((golden_on != golden_off).any(1).sum().item())
    return r


def run_campaign(runner: Runner, n_trials: int, seed: int, fault_model: int, rank: int = 0, world: int = 1,
                 group=None, prompt_seed: int = 7) -> CampaignResult:
    """This rank's share of n_trials (batches of runner.B rows), counters summed over ranks."""
    t0, t1 = trial_range(n_trials, world, rank)
    total = CampaignResult()
    gen = torch.Generator().manual_seed(prompt_seed)
    prompts = torch.randint(0, runner.cfg.vocab, (runner.B, runner.T), generator=gen).to(runner.device)
    t = t0
    while t < t1:
        res = run_batch(runner, prompts, seed, t, fault_model)
        take = min(runner.B, t1 - t)
        if take < runner.B:   # partial last batch: only count the first `take` rows
            res = _recount_partial(runner, prompts, seed, t, fault_model, take)
        total.add(res)
        t += runner.B
    if world > 1:
        import torch.distributed as dist
        v = total.as_tensor(runner.device)
        dist.all_reduce(v, group=group)
        total = CampaignResult.from_tensor(v)
    return total


def _recount_partial(runner, prompts, seed, trial0, fault_model, take):
    B, G = runner.B, runner.G
    widths = runner.cfg.linear_widths()
    sites = F2.make_fault_sites(seed, trial0, B, fault_model, widths, n_steps=G - 1, prompt_len=runner.T,
                                device=prompts.device)
    runner.sites = None
    g_off = runner.generate(prompts, "off", use_graph=False).clone()
    g_on = runner.generate(prompts, "fused", use_graph=False).clone()
    runner.sites = sites
    f_off = runner.generate(prompts, "off", use_graph=False).clone()
    f_on = runner.generate(prompts, "fused", use_graph=False).clone()
    corr = (runner.state.corrected.sum(0) + runner.state.nonfinite.sum(0))[:take]
    runner.sites = None
    r = CampaignResult()
    r.trials = take
    r.sdc_off = int((f_off != g_off)[:take].any(1).sum().item())
    r.sdc_on = int((f_on != g_on)[:take].any(1).sum().item())
    r.detected_on = int((corr > 0).sum().item())
    r.golden_mismatch = int((g_on != g_off)[:take].any(1).sum().item())
    return r
