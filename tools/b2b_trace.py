"""Per-launch CTA timeline of the back-to-back graph the bench's roofline
times: the 72 critical-layer GEMMs of one OPT-1.3B decode step (v/out
2048x2048, fc2 2048x8192; M = 32; CHECK, static weights) in one CUDA graph.
Needs lib/libft2_trace.so (python -m paper_conf_hpdc_sunzmg00y25_b200.build
--trace).  Prints, per launch: CTA count, first/last CTA start, median first
data, median MMA done, last CTA end (us from the graph's first CTA start), and
the gap between consecutive launches' last end."""
import ctypes, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CLK = bool(os.environ.get("CLOCK"))   # libft2_trace_clk.so: slots hold %clock64 (SM cycles)
NOTRACE = os.environ.get("NOTRACE") == "1"   # the product library: timing line only
os.environ["FT2_LIB"] = os.path.join(ROOT, "paper_conf_hpdc_sunzmg00y25_b200", "lib",
                                     os.environ.get("LIBNAME", "libft2.so") if NOTRACE else ("libft2_trace_clk.so" if CLK else "libft2_trace.so"))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
from paper_conf_hpdc_sunzmg00y25_b200 import _lib
import ft2_synth

L = _lib.load()
if not NOTRACE:
  L.ft2_debug_trace_read.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
  L.ft2_debug_trace_reset.argtypes = [ctypes.c_int]
M = int(os.environ.get("M", "32"))
NBLK = int(os.environ.get("NBLK", "8"))
shapes = [tuple(map(int, s.split("x"))) for s in os.environ.get("SHAPES", "2048x2048,2048x2048,2048x8192").split(",")]
dev = "cuda"
launches = []
xs = {}
SAMEW = os.environ.get("SAMEW") == "1"   # every launch of a shape reuses one weight tensor (L2-resident)
wcache = {}
for blk in range(NBLK):
    for j, (N, K) in enumerate(shapes):
        if SAMEW and (N, K) in wcache:
            w = wcache[(N, K)]
        else:
            w = ft2_synth.gen_bf16_torch((N, K), 100 + 8 * blk + j, 1, scale_log2=-6, device=dev)
            wcache[(N, K)] = w
        b = ft2_synth.gen_bf16_torch((N,), 300 + 8 * blk + j, 1, device=dev)
        if K not in xs:
            xs[K] = ft2_synth.gen_bf16_torch((M, K), 77, K, device=dev)
        launches.append((xs[K], w, b, torch.empty((M, N), dtype=torch.bfloat16, device=dev)))
big = torch.tensor([[-3.0e38, 3.0e38]], dtype=torch.bfloat16, device=dev).expand(M, 2).contiguous()
cnt = torch.zeros(M, dtype=torch.int32, device=dev)
mode = int(os.environ.get("MODE", str(1 | 16)))


PF = os.environ.get("PF", "0") == "1"   # pass the next launch's weights as the L2 prefetch hint


def run_all():
    for i, (x, w, b, y) in enumerate(launches):
        nxt = launches[(i + 1) % len(launches)][1] if PF else None
        ft2.protect_fused_gemm(x, w, y, bias=b, mode=mode, bounds=big, num_seqs=M, corrected_count=cnt,
                               l2_prefetch=nxt)


run_all()
torch.cuda.synchronize()
if not NOTRACE:
    L.ft2_debug_trace_reset(0)
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    run_all()
for _ in range(5):
    g.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    g.replay()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 10
nbytes = sum(w.numel() * 2 + x.numel() * 2 + y.numel() * 2 + b.numel() * 2 for x, w, b, y in launches)
print(f"graph of {len(launches)} launches: {1000 * ms / len(launches):.2f} us/launch, "
      f"{nbytes / (ms / 1e3) / 1e9:.0f} GB/s algorithmic", flush=True)
if NOTRACE:
    sys.exit(0)
g.replay()
torch.cuda.synchronize()
buf = np.zeros(32768 * 16, np.uint64)
L.ft2_debug_trace_read(buf.ctypes.data, buf.nbytes)
t = buf.reshape(128, 256, 16).astype(np.int64)
# slot 10 = SM id + 1: how many CTAs of one launch share an SM (and its tensor pipe)
occ = {}
for i in range(len(launches)):
    sm = t[i % 128][:, 10]
    sm = sm[sm > 0] - 1
    if sm.size == 0:
        continue
    per_sm = np.bincount(sm, minlength=148)
    h = np.bincount(per_sm, minlength=4)[:4]
    occ.setdefault(tuple(launches[i][1].shape), []).append((sm.size, int((per_sm > 0).sum()), int(h[2] + h[3:].sum())))
for k, v in occ.items():
    a = np.array(v)
    print(f"SM sharing {k[0]}x{k[1]}: CTAs {int(np.median(a[:, 0]))}, SMs used {np.median(a[:, 1]):.0f}, "
          f"SMs with >= 2 CTAs of the launch {np.median(a[:, 2]):.0f} (median over launches)")
if CLK:
    # per-CTA SM-cycle deltas from the moment its producer's PDL wait returned
    # (slot 2), medians over the CTAs of every launch of a shape
    sl = [0, 1, 2, 3, 12, 13, 4, 5, 14, 8, 9, 6, 15, 11, 7]
    per = {}
    for i in range(len(launches)):
        r = t[i % 128]
        r = r[(r[:, 0] > 0) & (r[:, 2] > 0) & (r[:, 7] > 0)]
        per.setdefault(tuple(launches[i][1].shape), []).append(r[:, sl] - r[:, 2:3])
    print("cycles after the CTA's PDL wait returned, median (p90) over CTAs; slots " + " ".join(map(str, sl)))
    for k, v in per.items():
        a = np.concatenate(v)
        print(f"{k[0]}x{k[1]:<6d}" + " ".join(f"{int(np.median(a[:, j])):6d}({int(np.percentile(a[:, j], 90)):5d})"
                                           for j in range(len(sl))))
    sys.exit(0)
# the last replay: rows whose start lies within the last graph's window
last_end = t[:, :, 7].max()
T0 = None
rows = []
for i in range(len(launches)):
    r = t[i % 128]
    r = r[r[:, 0] > last_end - int(2e6 * ms)]
    if r.shape[0] == 0:
        continue
    rows.append((i, r))
T0 = min(r[:, 0].min() for _, r in rows)
prev_end = None
spans = []
print(" i  shape        ctas  start0 startN  data_med mma_med  end_max   span  gap_from_prev_end")
for i, r in rows:
    N, K = launches[i][1].shape
    st0, stN = (r[:, 0].min() - T0) / 1e3, (r[:, 0].max() - T0) / 1e3
    dm = (np.median(r[r[:, 3] > 0, 3]) - T0) / 1e3 if (r[:, 3] > 0).any() else float("nan")
    mm = (np.median(r[r[:, 4] > 0, 4]) - T0) / 1e3 if (r[:, 4] > 0).any() else float("nan")
    en = (r[:, 7].max() - T0) / 1e3
    gap = en - prev_end if prev_end is not None else float("nan")
    spans.append(en - st0)
    if i < 12 or i >= len(rows) - 3:
        print(f"{i:2d} {N:5d}x{K:<5d} {r.shape[0]:5d} {st0:7.2f} {stN:6.2f} {dm:8.2f} {mm:7.2f} {en:8.2f} {en - st0:6.2f} {gap:6.2f}")
    prev_end = en
print(f"mean span per launch {np.mean(spans):.2f} us; last end {prev_end:.2f} us over {len(rows)} launches "
      f"= {prev_end / len(rows):.2f} us/launch")
# steady state per shape: median over launches of each slot's CTA median, relative
# to the previous launch's last CTA end (slots: 0 start 1 producer 2 x_wait_done
# 3 first_full 4 mma_issued 5 acc_ready 8 pushed 9 bar 6 recv_done 11 summed 7 done)
sl = [0, 1, 2, 3, 4, 5, 8, 9, 6, 11, 7]
per = {}
prev = None
for i, r in rows:
    if prev is not None and i >= 3:
        key = tuple(launches[i][1].shape)
        v = []
        for s_ in sl:
            c = r[r[:, s_] > 0, s_]
            v.append((np.median(c) - prev) / 1e3 if c.size else float("nan"))
        v.append((r[:, 7].max() - prev) / 1e3)
        per.setdefault(key, []).append(v)
    prev = r[:, 7].max()
print("slot medians rel. to previous launch end (us): " + " ".join(f"{x:>6}" for x in [str(s_) for s_ in sl] + ["end"]))
for k, v in per.items():
    print(f"{k[0]}x{k[1]:<6d}" + " ".join(f"{x:6.2f}" for x in np.median(np.array(v), axis=0)))
