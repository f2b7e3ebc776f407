"""Prefill-shaped (compute-bound) critical-layer GEMM: FT2 tcgen05 kernel
(PLAIN orientation A = x) vs cuBLAS, plus cuBLAS + the FT2 bound sweep (what
the runner does in prefill today).  TFLOP/s from 2*M*N*K.  CUDA graph of R
launches with rotated weights.  python tools/prefill_gemm_probe.py"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2

R = int(os.environ.get("R", 20))
shapes = [(4096, 2048, 2048), (4096, 2048, 8192), (4096, 4096, 4096), (4096, 11008, 4096), (4096, 4096, 11008),
          (512, 4096, 4096), (512, 11008, 4096), (512, 4096, 11008)]
if os.environ.get("SMALL"):
    shapes = [s for s in shapes if s[0] <= 512]
for M, N, K in shapes:
    ws = [ft2_synth.gen_bf16_torch((N, K), 21 + i, 1, scale_log2=-6, device="cuda") for i in range(4)]
    x = ft2_synth.gen_bf16_torch((M, K), 20, 1, device="cuda")
    b = ft2_synth.gen_bf16_torch((N,), 22, 1, device="cuda")
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    B = 32
    so = torch.arange(0, M + 1, M // B, dtype=torch.int32, device="cuda")
    bnd = torch.zeros((B, 2), dtype=torch.bfloat16, device="cuda")
    wsp = ft2.make_workspace(B)
    out = {"M": M, "N": N, "K": K}
    for kind in ("cublas", "ft2_plain", "cublas+bounds", "ft2_derive"):
        def run():
            for i in range(R):
                w = ws[i % 4]
                if kind.startswith("cublas"):
                    torch.addmm(b, x, w.t(), out=y)
                    if kind == "cublas+bounds":
                        ft2.bounds_from_prefill(y, bnd, wsp, seq_offsets=so, num_seqs=B, correct_nonfinite=True)
                elif kind == "ft2_derive":
                    ft2.prefill_fused_gemm(x, w, y, bnd, wsp, bias=b, seq_offsets=so, num_seqs=B)
                else:
                    ft2.protect_fused_gemm(x, w, y, bias=b, mode=0)
        run(); torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            run()
        g.replay(); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1000 / R
        out[kind + "_us"] = round(us, 2)
        out[kind + "_TFs"] = round(2 * M * N * K / us / 1e6, 1)
    print(json.dumps(out), flush=True)
