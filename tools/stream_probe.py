"""Effective HBM streaming rate of the decode GEMM's weight access pattern:
M = 32 swap-AB GEMMs with large weights (rotated copies > L2), CUDA events,
against a torch read of the same bytes (sum) and a copy."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
import ft2_synth


def t(fn, R=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(R):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / R


M = 32
for N, K in [(2048, 65536), (16384, 8192), (8192, 16384), (2048, 2048 * 16)]:
    ws = [ft2_synth.gen_bf16_torch((N, K), 30 + i, 1, scale_log2=-8, device="cuda") for i in range(2)]
    x = ft2_synth.gen_bf16_torch((M, K), 3, 1, device="cuda")
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    bnd = torch.tensor([[-1e30, 1e30]], dtype=torch.bfloat16, device="cuda")
    it = [0]

    def g():
        it[0] += 1
        ft2.protect_fused_gemm(x, ws[it[0] % 2], y, mode=1 | 16, bounds=bnd, num_seqs=1)

    def cub():
        it[0] += 1
        torch.matmul(x, ws[it[0] % 2].t(), out=y)

    def rd():
        it[0] += 1
        ws[it[0] % 2].view(torch.int16).sum(dtype=torch.int32)
    nb = N * K * 2
    for name, fn in (("ft2", g), ("cublas", cub), ("torch_sum", rd)):
        ms = t(fn)
        print(f"N={N} K={K} {name:10s} {ms * 1e3:8.1f} us  {nb / ms / 1e6:7.0f} GB/s", flush=True)
    del ws
    torch.cuda.empty_cache()
