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
# round 2: 128-row tiles (BA=64 is the default for these shapes), and site
# lists that overflow (100 directed sites in one row / tile -> the rescan path)
import numpy as _np
for (M, N, K) in [(32, 512, 512), (200, 512, 256)]:
    x = ft2_synth.gen_bf16_torch((M, K), 12, 1, device=dev)
    w = ft2_synth.gen_bf16_torch((N, K), 13, 1, scale_log2=-4, device=dev)
    out = torch.empty((M, N), dtype=torch.bfloat16, device=dev)
    raw = _np.zeros(100, [("trial", "<u4"), ("step", "<u2"), ("layer", "<u2"), ("token", "<u4"), ("col", "<u4"),
                          ("xor_mask", "<u4"), ("model", "u1"), ("nbits", "u1"), ("pad", "u1", (2,))])
    raw["step"], raw["col"], raw["xor_mask"] = (1 if M <= 128 else 0), (_np.arange(100) * 7) % 128, 1
    dsites = torch.from_numpy(raw.view(_np.uint8).copy()).to(dev)
    base = torch.zeros(100, dtype=torch.int32, device=dev)
    ft2.protect_fused_gemm(x, w, out, mode=1, bounds=torch.tensor([[-0.3, 0.3]], dtype=torch.bfloat16, device=dev),
                           num_seqs=1, sites=dsites, n_sites=100, cur_layer=0, cur_step=(1 if M <= 128 else 0),
                           base_row=base)
# FP32 variants (bounds with correction, protect, inject)
y32 = torch.randn((48, 260), device=dev)
y32.view(-1)[::37] = float("nan")
y32.view(-1)[5::53] = float("inf")
b32 = torch.zeros((4, 2), dtype=torch.float32, device=dev)
so32 = torch.tensor([0, 10, 10, 30, 48], dtype=torch.int32, device=dev)
ft2.bounds_from_prefill(y32, b32, ft2.make_workspace(4), seq_offsets=so32, num_seqs=4, correct_nonfinite=True,
                        keys_out=k)
ft2.bounds_finalize(k, b32)
ft2.protect(y32, b32, row_to_seq=(torch.arange(48, device=dev) % 4).to(torch.int32), num_seqs=4, corrected_count=cnt)
s32 = ft2.make_fault_sites(1, 0, 48, 0, [260], 4, 8, dtype=2)
ft2.inject_faults(y32, s32, 0, 2)
# persistent kernel with the (opt-in) K split, and DERIVE
os.environ["FT2_PREFILL_SPLITS"] = "2"
for (M, N, K) in [(256, 512, 1024), (136, 264, 1024)]:
    x = ft2_synth.gen_bf16_torch((M, K), 6, 1, device=dev)
    w = ft2_synth.gen_bf16_torch((N, K), 7, 1, scale_log2=-5, device=dev)
    out = torch.empty((M, N), dtype=torch.bfloat16, device=dev)
    ft2.protect_fused_gemm(x, w, out, mode=0)
    sq = torch.tensor([0, M // 2, M], dtype=torch.int32, device=dev)
    bd = torch.zeros((2, 2), dtype=torch.bfloat16, device=dev)
    ft2.prefill_fused_gemm(x, w, out, bd, ft2.make_workspace(2), seq_offsets=sq, num_seqs=2)
os.environ.pop("FT2_PREFILL_SPLITS")
# fused row-parallel all-reduce + check at P = 1 (handshake skipped) through the C ABI directly
# (round 2 session e: pointer tables are host arrays; also in place, y aliasing the partial)
fl = torch.zeros(1, dtype=torch.int32, device=dev)
words = torch.zeros(3, dtype=torch.int32, device=dev)
yo = torch.empty_like(yd)
ft2.allreduce_protect([yd.data_ptr()], 520, 1, 0, [fl.data_ptr()], words, yo, mode=1, bounds=b[:1].clone(),
                      num_seqs=1, corrected_count=cnt)
ft2.allreduce_protect([yo.data_ptr()], 520, 1, 0, [fl.data_ptr()], words, yo, mode=1,
                      bounds=torch.tensor([[-0.05, 0.05]], dtype=torch.bfloat16, device=dev), num_seqs=1,
                      corrected_count=cnt)
# round 2 session e: the default prefill K split (distributed reduction) at a 512-token shape
for (M, N, K) in [(512, 1024, 2048)]:
    x = ft2_synth.gen_bf16_torch((M, K), 8, 1, device=dev)
    w = ft2_synth.gen_bf16_torch((N, K), 9, 1, scale_log2=-5, device=dev)
    out = torch.empty((M, N), dtype=torch.bfloat16, device=dev)
    ft2.protect_fused_gemm(x, w, out, mode=0)
    sq = torch.arange(0, M + 1, M // 8, dtype=torch.int32, device=dev)
    bd = torch.zeros((8, 2), dtype=torch.bfloat16, device=dev)
    ft2.prefill_fused_gemm(x, w, out, bd, ft2.make_workspace(8), seq_offsets=sq, num_seqs=8)
torch.cuda.synchronize()
print("sanitize cases: done")
