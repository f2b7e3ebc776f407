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
# FP32 variants on the same bytes ([rows, n/2] fp32) and the fused
# row-parallel all-reduce + check at P = 1 on a decode-sized [32, 5120] layer
y32 = ft2_synth.gen_bf16_torch((rows, n // 2), 11, 5, device="cuda").float()
b32 = torch.zeros((32, 2), dtype=torch.float32, device="cuda")
w32 = torch.tensor([[-3e38, 3e38]], dtype=torch.float32, device="cuda")
for name, fn in [("bounds32_32seq", lambda: ft2.bounds_from_prefill(y32, b32, ws, seq_offsets=so, num_seqs=32)),
                 ("protect32", lambda: ft2.protect(y32, w32, corrected_count=cnt))]:
    for _ in range(3): fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(R): fn()
    e1.record(); torch.cuda.synchronize()
    us = 1000 * e0.elapsed_time(e1) / R
    out[name] = {"us": round(us, 2), "GBs": round(rows * n * 2 / us / 1e3, 1)}
if os.environ.get("AR", "1") == "1":
    import socket
    import torch.distributed as dist
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    s_ = socket.socket(); s_.bind(("127.0.0.1", 0))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(s_.getsockname()[1])); s_.close()
    dist.init_process_group("gloo", rank=0, world_size=1)
    rpc = tp.RowParallelCheck(32, 5120)
    yo = torch.empty((32, 5120), dtype=torch.bfloat16, device="cuda")
    bd = torch.tensor([[-3e38, 3e38]], dtype=torch.bfloat16, device="cuda").repeat(32, 1)
    c32 = torch.zeros(32, dtype=torch.int32, device="cuda")
    for i in range(4):
        rpc(i, yo, mode=1, bounds=bd, num_seqs=32, corrected_count=c32)
    torch.cuda.synchronize()
    dist.destroy_process_group()
print(json.dumps(out))
