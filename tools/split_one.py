"""One persistent-kernel GEMM at a small-M shape (for ncu): M N K from argv."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
M, N, K = (int(v) for v in sys.argv[1:4])
x = ft2_synth.gen_bf16_torch((M, K), 1, 1, device="cuda")
w = ft2_synth.gen_bf16_torch((N, K), 2, 1, scale_log2=-6, device="cuda")
y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
if os.environ.get("DERIVE"):
    S = 32
    so = torch.arange(0, M + 1, M // S, dtype=torch.int32, device="cuda")
    bnd = torch.zeros((S, 2), dtype=torch.bfloat16, device="cuda")
    wsp = ft2.make_workspace(S)
    for _ in range(3):
        ft2.prefill_fused_gemm(x, w, y, bnd, wsp, seq_offsets=so, num_seqs=S)
else:
    for _ in range(3):
        ft2.protect_fused_gemm(x, w, y, mode=0)
torch.cuda.synchronize()
