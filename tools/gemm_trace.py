"""Per-CTA timeline of one fused-GEMM launch (needs lib/libft2_trace.so:
python -m paper_conf_hpdc_sunzmg00y25_b200.build --trace).  The GEMM runs
right after a torch kernel (as in the decode runner) inside a CUDA graph."""
import ctypes, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ["FT2_LIB"] = os.path.join(ROOT, "paper_conf_hpdc_sunzmg00y25_b200", "lib", "libft2_trace.so")
sys.path.insert(0, ROOT)
import numpy as np
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
from paper_conf_hpdc_sunzmg00y25_b200 import _lib
import ft2_synth

L = _lib.load()
L.ft2_debug_trace_read.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
names = ["start", "prologue_done", "x_wait_done", "first_data", "mma_done", "acc_ready", "finish_start", "finish_done"]
shapes = [(32, 2048, 2048), (32, 4096, 4096), (32, 2048, 8192), (32, 11008, 4096)]
if len(sys.argv) > 3:
    a = list(map(int, sys.argv[1:])); shapes = [tuple(a[i:i + 3]) for i in range(0, len(a), 3)]
for M, N, K in shapes:
    x0 = ft2_synth.gen_bf16_torch((M, K), 20, 1, device="cuda")
    w = ft2_synth.gen_bf16_torch((N, K), 21, 1, scale_log2=-6, device="cuda")
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    bnd = torch.tensor([[-1e30, 1e30]], dtype=torch.bfloat16, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    nflush = int(os.environ.get("NOFLUSH", "0")) == 0
    big = [ft2_synth.gen_bf16_torch((N, K), 40 + i, 1, scale_log2=-6, device="cuda") for i in range(4)] if not nflush else []
    it = [0]
    def step():
        if nflush:
            flush.zero_()            # evict W from L2 (as a 2.6 GB weight stream would)
        else:                        # stream other weights through L2 with a read-only GEMM (no dirty lines)
            torch.matmul(x0[:, :64], big[it[0] % 4][:, :64].t())
            it[0] += 1
        x = torch.relu(x0)           # the preceding torch kernel
        ft2.protect_fused_gemm(x, w, y, mode=1 | 16, bounds=bnd, num_seqs=1)
    for _ in range(3): step()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    for _ in range(5): g.replay()
    torch.cuda.synchronize()
    buf = np.zeros(32768 * 16, np.uint64)
    L.ft2_debug_trace_read(buf.ctypes.data, buf.nbytes)
    t = buf.reshape(-1, 16).astype(np.int64)
    t = t[t[:, 0] > 0]
    clock = os.environ.get("FT2_TRACE_CLOCK")
    if clock:   # per-SM cycle counters: report each CTA relative to its own start, in us at 1.965 GHz
        t = t[t[:, 0] > 0]
        t = np.where(t > 0, t - t[:, :1], 0) + 1
        t0 = 1
        t = (t.astype(np.float64) / 1.965).astype(np.int64) + 1
    else:
        t0 = t[:, 0].max() - 200000   # ignore stale rows from earlier shapes
        t = t[t[:, 0] > t0]
        t0 = t[:, 0].min()
    buf[:] = 0
    L.ft2_debug_trace_write_zero() if hasattr(L, "ft2_debug_trace_write_zero") else None
    print(f"== M={M} N={N} K={K}: {t.shape[0]} CTAs; kernel span {(t[:, 7].max() - t0) / 1000:.2f} us")
    st = (t[:, 0] - t0) / 1000.0
    print(f"   start-time histogram (us): {np.histogram(st, bins=8)[0].tolist()} edges {np.round(np.histogram(st, bins=8)[1], 2).tolist()}")
    for j, n in enumerate(names):
        v = (t[:, j] - t0) / 1000.0
        v = v[t[:, j] > 0]
        if v.size:
            print(f"   {n:16s} min {v.min():6.2f}  med {np.median(v):6.2f}  max {v.max():6.2f} us")
