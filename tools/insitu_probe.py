"""In-situ decode GEMM probe: a CUDA graph of [torch layer_norm -> linear] pairs,
the pattern of a decode step (a host-model kernel precedes every critical
linear layer, so PDL cannot overlap the GEMM with a previous GEMM).  Compares
cuBLAS (F.linear) with the FT2 tcgen05 GEMM (PLAIN / CHECK) at the OPT-1.3B
critical shapes.  Weights are rotated beyond L2.

python tools/insitu_probe.py          (env R = pairs per graph, default 72)
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torch.nn.functional as F

import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2

M = int(os.environ.get("M", 32))
R = int(os.environ.get("R", 72))
shapes = [(2048, 2048), (2048, 2048), (2048, 8192)]   # v_proj, out_proj, fc2 of one OPT-1.3B block
if len(sys.argv) > 2:
    a = list(map(int, sys.argv[1:]))
    shapes = [tuple(a[i:i + 2]) for i in range(0, len(a), 2)]
dev = "cuda"
layers = []
for i in range(R):
    N, K = shapes[i % len(shapes)]
    w = ft2_synth.gen_bf16_torch((N, K), 100 + i, 1, scale_log2=ft2_synth.weight_scale_log2(K), device=dev)
    b = ft2_synth.gen_bf16_torch((N,), 300 + i, 1, device=dev)
    x = ft2_synth.gen_bf16_torch((M, K), 500 + (K % 97), 1, device=dev)
    y = torch.empty((M, N), dtype=torch.bfloat16, device=dev)
    lnw = torch.ones(K, dtype=torch.bfloat16, device=dev)
    layers.append((w, b, x, y, lnw))
bnd = torch.tensor([[-3e38, 3e38]], dtype=torch.bfloat16, device=dev).repeat(M, 1)
cnt = torch.zeros(M, dtype=torch.int32, device=dev)
wbytes = sum(w.numel() * 2 for w, *_ in layers)


HOST_NORM = os.environ.get("LN", "torch") == "ft2"   # LN=ft2: libft2's PDL-triggering host norm


def norm(x, lnw):
    if HOST_NORM:
        return ft2.host_norm(x, lnw, torch.empty_like(x), eps=1e-5)
    return F.layer_norm(x, (x.shape[1],), lnw, None, 1e-5)


def step(kind, with_ln=True):
    for w, b, x, y, lnw in layers:
        h = norm(x, lnw) if with_ln else x
        if kind == "cublas":
            torch.addmm(b, h, w.t(), out=y)
        else:
            mode = (1 if kind == "check" else 0) | (16 if os.environ.get("WSTATIC", "1") == "1" else 0)
            ft2.protect_fused_gemm(h, w, y, bias=b, mode=mode, bounds=bnd, num_seqs=M, corrected_count=cnt)


out = {"ln": "ft2" if HOST_NORM else "torch", "M": M, "pairs": R, "shapes": shapes, "weights_MB": round(wbytes / 1e6, 1)}
for with_ln in (True, False):
    for kind in ("cublas", "plain", "check", "ln_only"):
        if kind == "ln_only" and not with_ln:
            continue
        fn = (lambda: [norm(x, lnw) for _, _, x, _, lnw in layers]) \
            if kind == "ln_only" else (lambda k=kind: step(k, with_ln))
        fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            fn()
        for _ in range(3):
            g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(10):
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1000 / R)
        ts.sort()
        out[("ln+" if with_ln else "") + kind + "_us"] = round(ts[len(ts) // 2], 3)
print(json.dumps(out), flush=True)
