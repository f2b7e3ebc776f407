"""Where does a request's time go?  OPT-1.3B runner, B=32, prompt 128, gen 60:
per-request CUDA-event time, host time of the generate() call, and the
prefill / decode phase split, with the first-token pass eager or graphed."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_hpdc_sunzmg00y25_b200.runner import CONFIGS, Runner

r = Runner(CONFIGS["opt-1.3b"], 32, 128, 60, seed=1)
prompt = torch.randint(0, 50272, (32, 128), device="cuda")
for gp in (True, False, True):
    r.graph_prefill = gp
    for m in ("fused", "off"):
        for _ in range(2):
            r.generate(prompt, m)
        torch.cuda.synchronize()
        ev, host = [], []
        for _ in range(5):
            a, b = torch.cuda.Event(True), torch.cuda.Event(True)
            t0 = time.perf_counter()
            a.record(); r.generate(prompt, m); b.record()
            host.append((time.perf_counter() - t0) * 1e3)
            ev.append((a, b))
        torch.cuda.synchronize()
        r.time_phases = True
        r.generate(prompt, m)
        pre, dec = r.phase_times()
        r.time_phases = False
        print(json.dumps({"graph_prefill": gp, "mode": m, "event_ms": [round(a.elapsed_time(b), 2) for a, b in ev],
                          "host_ms": [round(h, 2) for h in host], "prefill_ms": round(pre, 2),
                          "decode_ms_per_step": round(dec, 4), "phase_sum_ms": round(pre + 59 * dec, 2)}), flush=True)
