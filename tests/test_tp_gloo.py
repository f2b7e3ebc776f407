"""Tensor-parallel bounds combine on CPU: world size 2 over gloo (SURVEY §4
tier 4a).  Each rank takes a column shard of a prefill output, computes its raw
keys with the oracle (test infrastructure), encodes them as the ABI does, and
the product's host logic (tp.allreduce_bounds_keys) combines them.  The
result must equal the unsharded oracle keys and bounds bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _encode(raw):
    # oracle raw keys (key(lo), key(hi)) -> ABI encoding (0xFFFF - key(lo), key(hi)); -1 stays -1
    enc = raw.copy()
    enc[:, 0] = np.where(raw[:, 0] >= 0, 0xFFFF - raw[:, 0], -1)
    return enc


def _worker(rank, world, port, out_q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import ft2_synth
    import oracle
    # the TP host logic lives in the product package, but importing the package
    # loads libft2.so; the module itself is pure torch.distributed
    import importlib.util
    spec = importlib.util.spec_from_file_location("ft2_tp", os.path.join(ROOT, "paper_conf_hpdc_sunzmg00y25_b200", "tp.py"))
    tp = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(tp)

    rows, n = 96, 640
    y = ft2_synth.plant_edge_values(ft2_synth.gen_bf16((rows, n), tau=9, sigma=77), stride=131, offset=5)
    so = np.array([0, 10, 10, 40, 96], np.int32)       # 4 sequences, one empty
    b, e = tp.column_shard(n, world, rank)
    shard = np.ascontiguousarray(y[:, b:e])
    _, raw, _ = oracle.bounds(shard, seq_offsets=so)
    keys = torch.from_numpy(_encode(raw))
    tp.allreduce_bounds_keys(keys)
    lo, hi = tp.decode_keys(keys)
    out_q.put((rank, keys.numpy().tolist(), lo.numpy().tolist(), hi.numpy().tolist()))
    dist.barrier()
    dist.destroy_process_group()


def test_tp_bounds_combine_world2():
    import ft2_synth
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    rows, n = 96, 640
    y = ft2_synth.plant_edge_values(ft2_synth.gen_bf16((rows, n), tau=9, sigma=77), stride=131, offset=5)
    so = np.array([0, 10, 10, 40, 96], np.int32)
    full_b, full_raw, _ = oracle.bounds(y.copy(), seq_offsets=so)
    for rank, keys, lo, hi in res:
        assert keys == _encode(full_raw).tolist()
        assert lo == full_raw[:, 0].tolist() and hi == full_raw[:, 1].tolist()
        # finalize of the combined keys equals the unsharded bounds
        assert oracle.bounds_from_keys(np.stack([lo, hi], 1)).tolist() == full_b.tolist()


def test_column_shard_partition():
    import importlib.util
    spec = importlib.util.spec_from_file_location("ft2_tp", os.path.join(ROOT, "paper_conf_hpdc_sunzmg00y25_b200", "tp.py"))
    tp = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(tp)
    for n in (5120, 13824, 7):
        for world in (1, 2, 4, 8):
            cols = []
            for r in range(world):
                b, e = tp.column_shard(n, world, r)
                cols.extend(range(b, e))
            assert cols == list(range(n))
