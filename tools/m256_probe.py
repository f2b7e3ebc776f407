"""Decode-GEMM routing probe for 128 < M <= 256 tokens (campaign batches):
CUDA graph of 8 launches over 8 rotated weight copies, cuBLAS vs FT2 CHECK.
Run with FT2_GEMM_SWAP_MAX=128 (persistent prefill kernel) and =256
(swap-AB decode kernel with 128-token tiles)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2

out = {"swap_max": os.environ.get("FT2_GEMM_SWAP_MAX", "128")}
for M in (192, 256):
    for N, K in ((4096, 4096), (11008, 4096), (4096, 11008)):
        ws = [ft2_synth.gen_bf16_torch((N, K), 40 + c, 1, scale_log2=-6, device="cuda") for c in range(8)]
        x = ft2_synth.gen_bf16_torch((M, K), 50, 1, device="cuda")
        y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        bnd = torch.tensor([[-3e38, 3e38]], dtype=torch.bfloat16, device="cuda").repeat(M, 1)
        cnt = torch.zeros(M, dtype=torch.int32, device="cuda")
        res = {}
        for kind in ("cublas", "check"):
            def body():
                for w in ws:
                    if kind == "cublas":
                        torch.mm(x, w.t(), out=y)
                    else:
                        ft2.protect_fused_gemm(x, w, y, mode=1 | 16, bounds=bnd, num_seqs=M, corrected_count=cnt)
            body()
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                body()
            for _ in range(3):
                g.replay()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(True), torch.cuda.Event(True)
            a.record()
            for _ in range(10):
                g.replay()
            b.record()
            torch.cuda.synchronize()
            res[kind] = round(a.elapsed_time(b) * 1000 / 80, 2)
        out[f"M{M}_{N}x{K}"] = res
        del ws
print(json.dumps(out), flush=True)
