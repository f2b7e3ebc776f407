"""Is the headline request host-bound?  Host time to enqueue one request
(prefill replay + 59 decode replays, no sync) against its GPU time, over
many requests, plus per-request GPU times (the bimodality of DESIGN.md §7)."""
import os, sys, time, json, statistics
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
from paper_conf_hpdc_sunzmg00y25_b200.runner import CONFIGS, Runner

r = Runner(CONFIGS["opt-1.3b"], 32, 128, 60, seed=1, device="cuda")
prompt = torch.randint(0, 50272, (32, 128), generator=torch.Generator().manual_seed(1)).cuda()
for _ in range(5):
    r.generate(prompt, "fused")
torch.cuda.synchronize()
host, gpu = [], []
t_end = time.time() + float(os.environ.get("SECS", "20"))
while time.time() < t_end:
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    a.record()
    t0 = time.perf_counter()
    r.generate(prompt, "fused")
    t1 = time.perf_counter()
    b.record()
    torch.cuda.synchronize()
    host.append(1000 * (t1 - t0))
    gpu.append(a.elapsed_time(b))
print(json.dumps({"requests": len(gpu), "gpu_ms": [round(x, 2) for x in gpu[::max(1, len(gpu) // 40)]],
                  "host_enqueue_ms": [round(x, 2) for x in host[::max(1, len(host) // 40)]],
                  "gpu_median": statistics.median(gpu), "host_median": statistics.median(host),
                  "host_us_per_graph_launch": 1000 * statistics.median(host) / r.G}))
