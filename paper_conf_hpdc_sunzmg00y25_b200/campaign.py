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
            "label": "proxy SDC = generated tokens differ from the golden run (random weights; not the paper's SDC)",
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
    g_on = runner.generate(prompt_ids, "fused", use_graph=use_graph).clone()
    g_corr = (runner.state.corrected.sum(0) + runner.state.nonfinite.sum(0)).clone()
    return g_off, g_on, g_corr


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
    golden_off, golden_on, golden_corr = golden if golden is not None else \
        golden_runs(runner, prompt_ids, use_graph, off_mode)
    runner.make_sites(seed, trial0, fault_model, step_policy=step_policy)
    faulty_off = runner.generate(prompt_ids, off_mode, use_graph=use_graph)[:take].clone()
    faulty_on = runner.generate(prompt_ids, "fused", use_graph=use_graph)[:take].clone()
    corrected = (runner.state.corrected.sum(0) + runner.state.nonfinite.sum(0))[:take]   # per trial row
    runner.set_sites(None)
    golden_off, golden_on, golden_corr = golden_off[:take], golden_on[:take], golden_corr[:take]
    r = CampaignResult()
    r.trials = take
    r.sdc_off = int((faulty_off != golden_off).any(1).sum().item())
    r.sdc_on = int((faulty_on != golden_on).any(1).sum().item())
    r.detected_on = int((corrected > golden_corr).sum().item())
    r.golden_mismatch = int((golden_on != golden_off).any(1).sum().item())
    r.fault_free_corrected = int((golden_corr > 0).sum().item())
    return r


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
