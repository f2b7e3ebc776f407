"""Bounds + check-and-clip kernels on the BASELINE full-size tensor
([65536, 11008] bf16 = 1.44 GB, Llama-2-7B prefill up_proj x 32 x 2048 tokens);
prints achieved GB/s (CUDA events, algorithmic 2 B/element)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
import ft2_synth

rows, n = int(os.environ.get("ROWS", 65536)), int(os.environ.get("COLS", 11008))
R = int(os.environ.get("R", 10))
y = ft2_synth.gen_bf16_torch((rows, n), 11, 5, device="cuda")
ws = ft2.make_workspace(32)
so = torch.arange(0, rows + 1, rows // 32, dtype=torch.int32, device="cuda")
b = torch.zeros((32, 2), dtype=torch.bfloat16, device="cuda")
wide = torch.tensor([[-3e38, 3e38]], dtype=torch.bfloat16, device="cuda")
cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
out = {"shape": [rows, n], "bytes": rows * n * 2}
for name, fn in [("bounds_32seq", lambda: ft2.bounds_from_prefill(y, b, ws, seq_offsets=so, num_seqs=32)),
                 ("protect", lambda: ft2.protect(y, wide, corrected_count=cnt))]:
    for _ in range(3): fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(R): fn()
    e1.record(); torch.cuda.synchronize()
    us = 1000 * e0.elapsed_time(e1) / R
    out[name] = {"us": round(us, 2), "GBs": round(rows * n * 2 / us / 1e3, 1)}
print(json.dumps(out))
