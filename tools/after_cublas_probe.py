"""Does our decode GEMM overlap a preceding cuBLAS GEMM (PDL)?  CUDA graph
of R pairs [cuBLAS k_proj-like GEMM -> v_proj-like GEMM (cuBLAS or FT2)] at
M = 32, 2048 x 2048, weights rotated beyond L2; per-pair us minus the cuBLAS
GEMM alone.  Also [torch relu -> GEMM] (no PDL trigger possible)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2

R = int(os.environ.get("R", 48))
N = K = int(os.environ.get("NK", 2048))
M = 32
wa = [ft2_synth.gen_bf16_torch((N, K), 100 + i, 1, scale_log2=-6, device="cuda") for i in range(R)]
wb = [ft2_synth.gen_bf16_torch((N, K), 300 + i, 1, scale_log2=-6, device="cuda") for i in range(R)]
x = ft2_synth.gen_bf16_torch((M, K), 5, 1, device="cuda")
ya = [torch.empty((M, N), dtype=torch.bfloat16, device="cuda") for _ in range(R)]
yb = [torch.empty((M, N), dtype=torch.bfloat16, device="cuda") for _ in range(R)]
bnd = torch.tensor([[-3e38, 3e38]], dtype=torch.bfloat16, device="cuda").repeat(M, 1)
cnt = torch.zeros(M, dtype=torch.int32, device="cuda")


def graph_time(fn):
    fn(); torch.cuda.synchronize()
    if os.environ.get("EAGER"):
        ts = []
        for _ in range(10):
            a, b = torch.cuda.Event(True), torch.cuda.Event(True)
            a.record(); fn(); b.record(); torch.cuda.synchronize()
            ts.append(a.elapsed_time(b) * 1000 / R)
        ts.sort()
        return round(ts[5], 3)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fn()
    for _ in range(3): g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(10):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(); g.replay(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1000 / R)
    ts.sort()
    return round(ts[5], 3)


def pre(kind, i):
    if kind == "cublas":
        torch.mm(x, wa[i].t(), out=ya[i])
    else:
        torch.relu(x, out=ya[i][:, :K] if N >= K else None) if False else ya[i].copy_(torch.relu(x[:, :N]) if N <= K else ya[i])


def second(kind, i):
    if kind == "cublas":
        torch.mm(x, wb[i].t(), out=yb[i])
    else:
        ft2.protect_fused_gemm(x, wb[i], yb[i], mode=1 | (16 if os.environ.get("WSTATIC", "1") == "1" else 0),
                               bounds=bnd, num_seqs=M, corrected_count=cnt)


out = {"M": M, "N": N, "K": K, "pairs": R}
for p in ("cublas", "relu"):
    out[f"{p}_alone"] = graph_time(lambda: [pre(p, i) for i in range(R)])
    for s in ("cublas", "ft2"):
        out[f"{p}+{s}"] = graph_time(lambda: [(pre(p, i), second(s, i)) for i in range(R)])
        out[f"{p}+{s}_net"] = round(out[f"{p}+{s}"] - out[f"{p}_alone"], 3)
print(json.dumps(out), flush=True)
