"""C5 campaign throughput probe: ms per decode step of the Llama-2-7B-shaped
runner at B=256 for golden (no sites) and faulty (sites armed) generations,
modes off / fused_plain / fused.  With PROFILE=1 it runs one faulty fused
generation inside an NVTX range 'c5_one' (for an ncu launch list)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_hpdc_sunzmg00y25_b200 import campaign
from paper_conf_hpdc_sunzmg00y25_b200.runner import CONFIGS, Runner

B = int(os.environ.get("B", 256))
model = os.environ.get("MODEL", "llama-2-7b")
r = Runner(CONFIGS[model], B, 16, 33, seed=1)
p = campaign.campaign_prompts(r)
out = {"B": B, "model": model}


def t(fn, n=3):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


if os.environ.get("PROFILE"):
    r.make_sites(1, 0, 2)
    for _ in range(2):
        r.generate(p, "fused")
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_push("c5_one")
    r.generate(p, "fused")
    torch.cuda.synchronize()
    torch.cuda.nvtx.range_pop()
    sys.exit(0)
r.time_phases = True
for faulty in (False, True):
    for mode in ("off", "fused_plain", "fused"):
        if faulty:
            r.make_sites(1, 0, 2)
        else:
            r.set_sites(None)
        ms = t(lambda: r.generate(p, mode))
        pre, dec = r.phase_times()
        out[f"{'faulty' if faulty else 'golden'}_{mode}"] = {"ms": round(ms, 3), "prefill_ms": round(pre, 3),
                                                             "decode_ms_per_step": round(dec, 3)}
print(json.dumps(out), flush=True)
