"""The bimodal request time: serve fused OPT-1.3B requests
back to back for SECS seconds; per request the GPU time, its prefill/decode
split, and NVML SM / memory clocks, power, temperature and throttle reasons
sampled right after it.  Prints one JSON line."""
import json, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import pynvml as N
from paper_conf_hpdc_sunzmg00y25_b200.runner import CONFIGS, Runner

N.nvmlInit()
h = N.nvmlDeviceGetHandleByIndex(0)
r = Runner(CONFIGS["opt-1.3b"], 32, 128, 60, seed=1, device="cuda")
prompt = torch.randint(0, 50272, (32, 128), generator=torch.Generator().manual_seed(1)).cuda()
for m in ("fused", "off"):
    for _ in range(3):
        r.generate(prompt, m)
torch.cuda.synchronize()
big_a = torch.empty(1 << 29, dtype=torch.bfloat16, device="cuda")
big_b = torch.empty_like(big_a)
wsmall = r.blocks[0].w["fc1"]
xs = torch.randn(32, 2048, device="cuda").to(torch.bfloat16)


def probe_kernels():
    """a 1 GB copy (GB/s) and 50 back-to-back cuBLAS 32x8192x2048 GEMMs on one
    weight (L2-resident, us each): which kinds of work the state slows"""
    e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    e[0].record(); big_b.copy_(big_a); e[1].record()
    for _ in range(50):
        torch.matmul(xs, wsmall.t())
    e[2].record()
    torch.cuda.synchronize()
    return round(2 * big_a.numel() * 2 / e[0].elapsed_time(e[1]) / 1e6), round(1000 * e[1].elapsed_time(e[2]) / 50, 2)


rows = []
kern = []
t_end = time.time() + float(os.environ.get("SECS", "120"))
r.time_phases = True
get_reasons = getattr(N, "nvmlDeviceGetCurrentClocksEventReasons", None) or N.nvmlDeviceGetCurrentClocksThrottleReasons
while time.time() < t_end:
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    r.generate(prompt, os.environ.get("MODE", "fused"))
    b.record()
    b.synchronize()
    pre, dec = r.phase_times()
    if len(rows) % 20 == 0:
        kern.append([round(time.time() - t_end, 1)] + list(probe_kernels()))
    rows.append([round(time.time() - t_end, 1), round(a.elapsed_time(b), 2), round(pre, 2), round(dec * 1000, 1),
                 N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM), N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_MEM),
                 round(N.nvmlDeviceGetPowerUsage(h) / 1e3), N.nvmlDeviceGetTemperature(h, 0), int(get_reasons(h))])
print(json.dumps({"cols": ["t_s", "ms", "prefill_ms", "decode_us_per_step", "sm_mhz", "mem_mhz", "power_w", "temp_c",
                           "reasons"], "rows": rows, "kernels_cols": ["t_s", "copy_GBps", "cublas_gemm_us"],
                  "kernels": kern}))
