"""Small cases of every kernel for compute-sanitizer (memcheck / racecheck / synccheck / initcheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
import ft2_synth

torch.manual_seed(0)
dev = "cuda"
# bounds (multi-seq, correction, overflow path) and protect
y = ft2_synth.plant_edge_values(ft2_synth.gen_bf16((64, 520), 1, 1), stride=7)
yd = torch.from_numpy(y.view(np.int16)).view(torch.bfloat16).to(dev)
so = torch.tensor([0, 10, 10, 40, 64], dtype=torch.int32, device=dev)
b = torch.zeros((4, 2), dtype=torch.bfloat16, device=dev)
k = torch.zeros((4, 2), dtype=torch.int32, device=dev)
ws = ft2.make_workspace(4)
ft2.bounds_from_prefill(yd, b, ws, seq_offsets=so, num_seqs=4, correct_nonfinite=True, keys_out=k)
cnt = torch.zeros(4, dtype=torch.int32, device=dev)
r2s = (torch.arange(64, device=dev) % 4).to(torch.int32)
ft2.protect(yd, b, row_to_seq=r2s, num_seqs=4, corrected_count=cnt)
ft2.bounds_finalize(k, b)
# sites + inject
s = ft2.make_fault_sites(1, 0, 64, 2, [520] * 3, 4, 8)
ft2.inject_faults(yd, s, 1, 2)
# fused GEMM: decode (split-K cluster), single split, prefill orientation, with sites and checks
for (M, N, K) in [(8, 384, 512), (32, 256, 128), (1, 200, 72), (160, 256, 192)]:
    x = ft2_synth.gen_bf16_torch((M, K), 2, 1, device=dev)
    w = ft2_synth.gen_bf16_torch((N, K), 3, 1, scale_log2=-4, device=dev)
    bias = ft2_synth.gen_bf16_torch((N,), 4, 1, device=dev)
    out = torch.empty((M, N), dtype=torch.bfloat16, device=dev)
    bb = torch.tensor([[-0.3, 0.3]], dtype=torch.bfloat16, device=dev)
    c = torch.zeros(1, dtype=torch.int32, device=dev)
    sites = ft2.make_fault_sites(5, 0, M, 0, [N], 2, 1)
    ft2.protect_fused_gemm(x, w, out, bias=bias, mode=1, bounds=bb, num_seqs=1, corrected_count=c, sites=sites,
                           cur_layer=0, cur_step=1)
    ft2.protect_fused_gemm(x, w, out, bias=bias, mode=0)
torch.cuda.synchronize()
print("sanitize cases: done")
