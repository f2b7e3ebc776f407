"""One PLAIN and one DERIVE launch of the prefill GEMM at the OPT-1.3B prefill
shape [4096 x 2048 x 2048], 32 sequences (for ncu captures)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
M, N, K, B = [int(v) for v in (sys.argv[1:5] if len(sys.argv) > 4 else (4096, 2048, 2048, 32))]
x = ft2_synth.gen_bf16_torch((M, K), 20, 1, device="cuda")
w = ft2_synth.gen_bf16_torch((N, K), 21, 1, scale_log2=-6, device="cuda")
b = ft2_synth.gen_bf16_torch((N,), 22, 1, device="cuda")
y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
so = torch.arange(0, M + 1, M // B, dtype=torch.int32, device="cuda")
bnd = torch.zeros((B, 2), dtype=torch.bfloat16, device="cuda")
ws = ft2.make_workspace(B)
for _ in range(2):
    ft2.protect_fused_gemm(x, w, y, bias=b, mode=0)
    ft2.prefill_fused_gemm(x, w, y, bnd, ws, bias=b, seq_offsets=so, num_seqs=B)
torch.cuda.synchronize()
