"""Split-K debug: compare the persistent kernel against cuBLAS per 128x256
half-tile and time it, for the split count in FT2_PREFILL_SPLITS."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2

out = {"splits_env": os.environ.get("FT2_PREFILL_SPLITS")}
for M, N, K in ((512, 11008, 4096), (256, 4096, 4096), (512, 4096, 4096)):
    x = ft2_synth.gen_bf16_torch((M, K), 1, 1, device="cuda")
    w = ft2_synth.gen_bf16_torch((N, K), 2, 1, scale_log2=-6, device="cuda")
    y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    ft2.protect_fused_gemm(x, w, y, mode=0)
    torch.cuda.synchronize()
    ref = (x.float() @ w.float().t())
    err = ((y.float() - ref).abs() > 1e-2 * ref.abs().clamp_min(1e-2)).float()
    bad = err.view(M // 128, 128, -1)
    nt = (N + 255) // 256
    badt = []
    for mt in range(M // 128):
        for nt_ in range(nt):
            v = bad[mt, :, nt_ * 256:(nt_ + 1) * 256].mean().item()
            if v > 0.01:
                badt.append((mt, nt_, round(v, 2)))
    for _ in range(3):
        ft2.protect_fused_gemm(x, w, y, mode=0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    for _ in range(20):
        ft2.protect_fused_gemm(x, w, y, mode=0)
    b.record()
    torch.cuda.synchronize()
    out[f"{M}x{N}x{K}"] = {"us": round(a.elapsed_time(b) * 50, 2), "ws_need": ft2.gemm_workspace_bytes(M, N, K),
                           "bad_tiles": badt[:40], "n_bad": len(badt)}
print(json.dumps(out), flush=True)
