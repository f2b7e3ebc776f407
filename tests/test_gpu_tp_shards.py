"""Tensor-parallel bounds on one GPU: a
column-parallel critical layer's prefill output is split into P column shards
(strided views of one tensor, as each TP rank would hold them), every shard
runs ft2_bounds_from_prefill(finalize=0, keys_out), the keys are combined with
the element-wise MAX the NCCL all-reduce performs (torch.maximum on the
device), and ft2_bounds_finalize produces the bounds.  They must equal the
unsharded oracle bounds bit for bit for every P (the multi-process version of
the same host logic runs on gloo in test_tp_gloo.py)."""
import numpy as np
import pytest
import torch

import ft2_synth
import oracle
from gpu_util import dev, dev_i32, host

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("P", [1, 2, 4, 8])
@pytest.mark.parametrize("n", [5120, 13824])   # Llama-2-13B v_proj / up_proj widths
def test_column_shards_combine_to_unsharded(P, n):
    import paper_conf_hpdc_sunzmg00y25_b200 as ft2
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    rows = 96
    y = ft2_synth.plant_edge_values(ft2_synth.gen_bf16((rows, n), tau=31, sigma=P), stride=389, offset=7)
    so = np.array([0, 16, 16, 50, 96], np.int32)     # 4 sequences, one empty
    want_b, want_raw, _ = oracle.bounds(y.copy(), seq_offsets=so)
    yd, sod = dev(y), dev_i32(so)
    S = so.size - 1
    keys = []
    for r in range(P):
        b, e = tp.column_shard(n, P, r)
        k = torch.empty((S, 2), dtype=torch.int32, device="cuda")
        ft2.bounds_from_prefill(yd[:, b:e], None, ft2.make_workspace(S), seq_offsets=sod, num_seqs=S,
                                finalize=False, keys_out=k)
        keys.append(k)
    comb = keys[0]
    for k in keys[1:]:
        comb = torch.maximum(comb, k)           # what all_reduce(MAX) computes
    bnd = torch.zeros((S, 2), dtype=torch.bfloat16, device="cuda")
    ft2.bounds_finalize(comb, bnd)
    assert np.array_equal(host(bnd), want_b)
    lo, hi = tp.decode_keys(comb.cpu())
    assert lo.numpy().tolist() == want_raw[:, 0].tolist() and hi.numpy().tolist() == want_raw[:, 1].tolist()


def test_tp_bounds_from_prefill_world1_nccl():
    """The product's TP entry point end to end over a real NCCL process group
    of size 1 (the all-reduce is the identity; the call path is the one
    torchrun ranks take)."""
    import os
    import socket
    import torch.distributed as dist
    import paper_conf_hpdc_sunzmg00y25_b200 as ft2
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        y = ft2_synth.gen_bf16((64, 2560), tau=5, sigma=3)
        so = np.array([0, 32, 64], np.int32)
        want_b, _, _ = oracle.bounds(y.copy(), seq_offsets=so)
        bnd = torch.zeros((2, 2), dtype=torch.bfloat16, device="cuda")
        tp.tp_bounds_from_prefill(dev(y), bnd, ft2.make_workspace(2), seq_offsets=dev_i32(so))
        torch.cuda.synchronize()
        assert np.array_equal(host(bnd), want_b)
    finally:
        dist.destroy_process_group()
