"""Time the fused GEMM alone at decode shapes vs cuBLAS (F.linear).  Usage:
python tools/gemm_probe.py [M N K ...]  (env FT2_GEMM_SPLITK forces split-K)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torch.nn.functional as F
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
import ft2_synth

shapes = [(32, 2048, 2048), (32, 2048, 8192), (32, 4096, 4096), (32, 11008, 4096), (32, 4096, 11008), (1, 2048, 2048)]
if len(sys.argv) > 3:
    a = list(map(int, sys.argv[1:]))
    shapes = [tuple(a[i:i + 3]) for i in range(0, len(a), 3)]
R = int(os.environ.get("R", "50"))
res = []
for M, N, K in shapes:
    copies = max(1, int(300e6 // (N * K * 2)) + 1)   # rotate weights beyond L2
    ws = [ft2_synth.gen_bf16_torch((N, K), 21 + i, 1, scale_log2=-6, device="cuda") for i in range(copies)]
    x = ft2_synth.gen_bf16_torch((M, K), 20, 1, device="cuda")
    b = ft2_synth.gen_bf16_torch((N,), 22, 1, device="cuda")
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    bnd = torch.tensor([[-1e30, 1e30]], dtype=torch.bfloat16, device="cuda")
    def run(kind, i):
        w = ws[i % copies]
        if kind == "cublas":
            torch.addmm(b, x, w.t(), out=y)
        else:
            ft2.protect_fused_gemm(x, w, y, bias=b, mode=(1 if kind == "check" else 0) | (16 if os.environ.get("WSTATIC", "1") == "1" else 0), bounds=bnd, num_seqs=1)
    out = {"M": M, "N": N, "K": K}
    for kind in ("cublas", "plain", "check"):
        for i in range(5):
            run(kind, i)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for i in range(R):
                run(kind, i)
        g.replay(); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
        us = 1000 * e0.elapsed_time(e1) / R
        out[kind + "_us"] = round(us, 2)
        out[kind + "_GBs"] = round((N * K * 2 + M * K * 2 + M * N * 2) / us / 1e3, 1)
    res.append(out)
    print(json.dumps(out), flush=True)
