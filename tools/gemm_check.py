"""Correctness sweep of the fused GEMM over shapes x forced split-K (env is read
once per process, so each split count runs in its own subprocess)."""
import os, subprocess, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 1 and sys.argv[1] == "child":
    import torch
    import paper_conf_hpdc_sunzmg00y25_b200 as ft2
    import ft2_synth
    for M, N, K in [(1, 2048, 2048), (1, 768, 768), (32, 2048, 2048), (16, 256, 1024), (1, 128, 1024)]:
        x = ft2_synth.gen_bf16_torch((M, K), 20, 1, device="cuda")
        w = ft2_synth.gen_bf16_torch((N, K), 21, 1, scale_log2=-5, device="cuda")
        y = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        ft2.protect_fused_gemm(x, w, y, mode=0)
        ref = (x.float() @ w.float().t())
        err = (y.float() - ref).abs() / ref.abs().clamp_min(1e-2)
        bad = (err > 2e-2)
        idx = bad.nonzero()[:, 1].unique().tolist()[:12] if bad.any() else []
        print(json.dumps({"sk": os.environ.get("FT2_GEMM_SPLITK"), "M": M, "N": N, "K": K,
                          "nbad": int(bad.sum()), "bad_cols": idx}), flush=True)
else:
    for sk in ["0", "1", "2", "3", "4", "6", "8", "9", "16"]:
        env = dict(os.environ, FT2_GEMM_SPLITK=sk)
        subprocess.run([sys.executable, __file__, "child"], env=env)
