"""Per-launch cost of ft2_allreduce_protect at P = 1 against ft2_protect on the
same [32, 5120] bf16 decode output: CUDA graphs of 80 back-to-back launches
(the row-parallel layers of one Llama-2-13B decode step), us per launch."""
import os, socket, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import torch.distributed as dist
import ft2_synth
import paper_conf_hpdc_sunzmg00y25_b200 as ft2
from paper_conf_hpdc_sunzmg00y25_b200 import tp

s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
dist.init_process_group("gloo", rank=0, world_size=1)
B, n, L = 32, 5120, 80
dev = "cuda"
rpc = tp.RowParallelCheck(B, n)
part = ft2_synth.gen_bf16_torch((B, n), 970, 5, device=dev)
rpc.partials[0].copy_(part); rpc.partials[1].copy_(part)
bias = ft2_synth.gen_bf16_torch((n,), 971, 5, device=dev)
bnd = torch.tensor([[-3.0e38, 3.0e38]], dtype=torch.bfloat16, device=dev).repeat(B, 1)
cnt = torch.zeros(B, dtype=torch.int32, device=dev)
ys = [torch.empty((B, n), dtype=torch.bfloat16, device=dev) for _ in range(L)]
bufs = [part.clone() for _ in range(L)]


def timed(fn, R=20):
    st = torch.cuda.Stream()
    st.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(st):
        fn()
    torch.cuda.current_stream().wait_stream(st)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fn()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(R):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    return 1000 * a.elapsed_time(b) / R / L


variants = {
    "protect": lambda: [ft2.protect(bufs[i], bnd, num_seqs=B, corrected_count=cnt) for i in range(L)],
    "protect_same_buf": lambda: [ft2.protect(bufs[0], bnd, num_seqs=B, corrected_count=cnt) for i in range(L)],
    "ar_inplace_check": lambda: [rpc(i, rpc.partial(i), mode=1, bounds=bnd, num_seqs=B, corrected_count=cnt) for i in range(L)],
    "ar_inplace_plain": lambda: [rpc(i, rpc.partial(i), mode=0) for i in range(L)],
    "ar_y_check": lambda: [rpc(i, ys[i], mode=1, bounds=bnd, num_seqs=B, corrected_count=cnt) for i in range(L)],
    "ar_y_bias_check": lambda: [rpc(i, ys[i], bias=bias, mode=1, bounds=bnd, num_seqs=B, corrected_count=cnt) for i in range(L)],
    "torch_copy": lambda: [ys[i].copy_(bufs[i]) for i in range(L)],
}
for k, fn in variants.items():
    print(f"{k:20s} {timed(fn):6.2f} us/launch", flush=True)
dist.destroy_process_group()
