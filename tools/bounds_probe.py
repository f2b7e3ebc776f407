"""Prefill-shaped bound sweeps (ft2_bounds_from_prefill) inside a CUDA graph:
R launches on distinct [rows, n] tensors (B sequences each), either right
after a torch kernel that writes the tensor (L2-warm, as after the layer's
GEMM in prefill) or on tensors rotated beyond L2 (cold).  Prints us/launch
and algorithmic GB/s (2 B/element).  python tools/bounds_probe.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2

R = int(os.environ.get("R", 72))
for rows, n, B in [(4096, 2048, 32), (4096, 2048, 1), (4096, 8192, 32), (512, 4096, 32), (65536, 11008, 32)]:
    nt = max(1, min(R, int(2e9 // (rows * n * 2))))
    ys = [ft2_synth.gen_bf16_torch((rows, n), 30 + i, 1, device="cuda") for i in range(min(nt, 8))]
    src = ys[0].clone()
    so = torch.arange(0, rows + 1, rows // B, dtype=torch.int32, device="cuda")
    bnd = torch.zeros((B, 2), dtype=torch.bfloat16, device="cuda")
    ws = ft2.make_workspace(B)
    nf = torch.zeros(B, dtype=torch.int32, device="cuda")
    out = {"shape": [rows, n], "seqs": B}
    for warm in (True, False):
        reps = R if rows * n < 1e8 else 4

        def body():
            for i in range(reps):
                y = ys[i % len(ys)]
                if warm:
                    y.copy_(src)
                ft2.bounds_from_prefill(y, bnd, ws, seq_offsets=so, num_seqs=B, correct_nonfinite=True,
                                        nonfinite_count=nf)

        def copies():
            for i in range(reps):
                ys[i % len(ys)].copy_(src)
        ts = {}
        for name, fn in (("all", body), ("copy", copies)):
            if name == "copy" and not warm:
                continue
            fn()
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                fn()
            g.replay()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
            ts[name] = e0.elapsed_time(e1) * 1000 / reps
        us = ts["all"] - ts.get("copy", 0.0)
        out["warm_us" if warm else "cold_us"] = round(us, 2)
        out["warm_GBs" if warm else "cold_GBs"] = round(rows * n * 2 / us / 1e3, 1)
    print(json.dumps(out), flush=True)
