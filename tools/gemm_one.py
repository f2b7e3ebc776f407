"""A few M=32 decode GEMMs (CHECK, static weights) of one shape, for ncu
captures: python tools/gemm_one.py N K [reps]"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
import ft2_synth

N, K = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 6
M = 32
ws = [ft2_synth.gen_bf16_torch((N, K), 30 + i, 1, scale_log2=-6, device="cuda") for i in range(4)]
x = ft2_synth.gen_bf16_torch((M, K), 3, 1, device="cuda")
b = ft2_synth.gen_bf16_torch((N,), 4, 1, device="cuda")
y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
bnd = torch.tensor([[-1e30, 1e30]], dtype=torch.bfloat16, device="cuda").expand(M, 2).contiguous()
cnt = torch.zeros(M, dtype=torch.int32, device="cuda")
for i in range(reps):
    ft2.protect_fused_gemm(x, ws[i % 4], y, bias=b, mode=1 | 16, bounds=bnd, num_seqs=M, corrected_count=cnt)
torch.cuda.synchronize()
