"""Launch-gap decomposition of one decode GEMM in situ (trace build,
lib/libft2_trace.so): graph = relu -> mark(0) -> GEMM -> mark(1), with the
GEMM either cuBLAS or the FT2 tcgen05 kernel; mark kernels record
%globaltimer.  Reports (mark1 - mark0) and, for FT2, the first CTA start and
last CTA end relative to mark 0.  python tools/gap_probe.py [N K]"""
import ctypes, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CLK = bool(os.environ.get("CLOCK"))   # libft2_trace_clk.so: slots hold %clock64 (cycles) instead of ns
os.environ["FT2_LIB"] = os.path.join(ROOT, "paper_conf_hpdc_sunzmg00y25_b200", "lib",
                                     "libft2_trace_clk.so" if CLK else "libft2_trace.so")
sys.path.insert(0, ROOT)
import numpy as np
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
from paper_conf_hpdc_sunzmg00y25_b200 import _lib
import ft2_synth

L = _lib.load()
L.ft2_debug_trace_read.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
L.ft2_debug_mark.argtypes = [ctypes.c_int, ctypes.c_void_p]
L.ft2_debug_marks_read.argtypes = [ctypes.c_void_p]
N, K = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (2048, 2048)
M = 32
ws = [ft2_synth.gen_bf16_torch((N, K), 21 + i, 1, scale_log2=-6, device="cuda") for i in range(8)]
x0 = ft2_synth.gen_bf16_torch((M, K), 20, 1, device="cuda")
b = ft2_synth.gen_bf16_torch((N,), 22, 1, device="cuda")
y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
bnd = torch.tensor([[-1e30, 1e30]], dtype=torch.bfloat16, device="cuda")


hot_a = torch.randn(4096, 4096, device="cuda", dtype=torch.bfloat16)


def mark(i):
    L.ft2_debug_mark(i, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))


for kind in ("cublas", "ft2", "none"):
    res = []
    for rep in range(8):
        w = ws[rep % 8]
        def step():
            x = torch.relu(x0)
            mark(0)
            if kind == "cublas":
                torch.addmm(b, x, w.t(), out=y)
            elif kind == "ft2":
                ft2.protect_fused_gemm(x, w, y, bias=b, mode=1 | 16, bounds=bnd, num_seqs=1)
            mark(1)
        step(); torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            step()
        for _ in range(3):
            g.replay()
        if os.environ.get("HOT"):     # keep the SM clock up: a busy GPU right before the measured replay
            for _ in range(int(os.environ.get("HOT"))):
                torch.matmul(hot_a, hot_a)
            g.replay()
        torch.cuda.synchronize()
        buf = np.zeros(32768 * 16, np.uint64)
        L.ft2_debug_trace_read(buf.ctypes.data, buf.nbytes)
        mk = np.zeros(64, np.uint64)
        L.ft2_debug_marks_read(mk.ctypes.data)
        m0, m1 = int(mk[0]), int(mk[1])
        t = buf.reshape(-1, 16).astype(np.int64)
        if CLK:
            if kind == "ft2" and rep == 7:
                t = t[t[:, 0] > 0]
                d = t[:, [0, 1, 2, 3, 4, 5, 8, 9, 10, 6, 11, 7]] - t[:, :1]
                print("cycles after CTA start, median over CTAs (slots 0 1 2 3 4 5 8 9 10 6 11 7):",
                      np.median(d, axis=0).astype(int).tolist())
            res.append({"total": (m1 - m0) / 1e3})
            continue
        t = t[(t[:, 0] >= m0) & (t[:, 0] <= m1)]
        r = {"total": (m1 - m0) / 1e3}
        if kind == "ft2" and t.shape[0]:
            r["first_start"] = (t[:, 0].min() - m0) / 1e3
            r["last_start"] = (t[:, 0].max() - m0) / 1e3
            r["first_data_med"] = (np.median(t[:, 3]) - m0) / 1e3
            r["mma_done_max"] = (t[:, 4].max() - m0) / 1e3
            r["finish_start_med"] = (np.median(t[:, 6]) - m0) / 1e3
            r["last_end"] = (t[:, 7].max() - m0) / 1e3
        res.append(r)
        if kind == "ft2" and rep == 7 and os.environ.get("DUMP"):
            o = np.argsort(t[:, 0])
            sl = [0, 1, 2, 3, 4, 5, 8, 9, 10, 6, 11, 7]
            print("cta  " + " ".join(f"{i:>6d}" for i in sl) + "   (us after mark 0; slots: 0 start 1 prologue 2 x_wait "
                  "3 first_data 4 mma_issued 5 acc_ready 8 pushed 9 named_bar 10 griddep 6 recv_done 11 summed 7 done)")
            for j in o:
                print(f"{j:4d} " + " ".join(f"{(t[j, i] - m0) / 1e3:6.2f}" if t[j, i] > 0 else "     -" for i in sl))
    keys = res[0].keys()
    print(kind, N, K, {k: round(float(np.median([r[k] for r in res])), 2) for k in keys}, flush=True)
