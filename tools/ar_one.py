"""One eager launch each of ft2_protect and ft2_allreduce_protect (P = 1, in
place, PLAIN / CHECK) on a [32, 5120] bf16 tensor, for an ncu capture."""
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
B, n = 32, 5120
rpc = tp.RowParallelCheck(B, n)
part = ft2_synth.gen_bf16_torch((B, n), 970, 5, device="cuda")
rpc.partials[0].copy_(part); rpc.partials[1].copy_(part)
bnd = torch.tensor([[-3.0e38, 3.0e38]], dtype=torch.bfloat16, device="cuda").repeat(B, 1)
cnt = torch.zeros(B, dtype=torch.int32, device="cuda")
buf = part.clone()
for r in range(3):
    ft2.protect(buf, bnd, num_seqs=B, corrected_count=cnt)
    rpc(2 * r, rpc.partial(2 * r), mode=0)
    rpc(2 * r + 1, rpc.partial(2 * r + 1), mode=1, bounds=bnd, num_seqs=B, corrected_count=cnt)
torch.cuda.synchronize()
dist.destroy_process_group()
