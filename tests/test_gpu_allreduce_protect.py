"""ft2_allreduce_protect: a row-parallel critical
layer's one-shot sum all-reduce over CUDA IPC peer memory fused with the check,
bit-exact against the oracle (reading A22 + R7 + R5), identical on every rank.
World size 2 runs as two processes sharing the one GPU (IPC mappings of the
same device; gloo exchanges the handles); P = 1 runs in-process."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import ft2_synth
import oracle

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ROWS, N, CALLS = 32, 5120, 5


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _inputs(i, world):
    parts = np.stack([ft2_synth.gen_bf16((ROWS, N), 300 + 16 * i + t, 9) for t in range(world)])
    bias = ft2_synth.gen_bf16((N,), 299, 9)
    rng = np.random.default_rng(i)
    bounds = np.stack([[oracle.f64_to_bf16(-abs(rng.normal(1.0, 0.3)) - 0.1),
                        oracle.f64_to_bf16(abs(rng.normal(1.0, 0.3)) + 0.1)] for _ in range(ROWS)]).astype(np.uint16)
    sites = oracle.make_sites(11, 64 * i, ROWS, oracle.FAULT_EXP, [N], n_steps=1, prompt_len=1, step_policy=1)
    return parts, bias, bounds, sites


def _worker(rank, world, port, q):
    import sys
    sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from gpu_util import dev, host, sites_to_dev
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    rpc = tp.RowParallelCheck(ROWS, N)
    out = []
    for i in range(CALLS):
        parts, bias, bounds, sites = _inputs(i, world)
        rpc.partial(i).copy_(dev(parts[rank]))
        y = torch.empty((ROWS, N), dtype=torch.bfloat16, device="cuda")
        cnt = torch.zeros(ROWS, dtype=torch.int32, device="cuda")
        torch.cuda.synchronize()
        rpc(i, y, bias=dev(bias), mode=1, bounds=dev(bounds), num_seqs=ROWS, corrected_count=cnt,
            sites=sites_to_dev(sites), n_sites=ROWS, cur_layer=0, cur_step=1)
        torch.cuda.synchronize()
        out.append((host(y).tobytes(), cnt.cpu().numpy().tolist()))
    q.put((rank, out, rpc.status()))
    dist.barrier()
    rpc.close()
    dist.destroy_process_group()


def _check(results, world):
    for i in range(CALLS):
        parts, bias, bounds, sites = _inputs(i, world)
        want, wcnt = oracle.allreduce_protect(parts, bias=bias, bounds_=bounds, sites=sites, cur_layer=0, cur_step=1)
        for rank, out, status in results:
            assert status == 0
            y = np.frombuffer(out[i][0], np.uint16).reshape(ROWS, N)
            assert np.array_equal(y, want), (rank, i)
            assert np.array_equal(np.array(out[i][1], np.uint32), wcnt), (rank, i)
        assert int(wcnt.sum()) > 0   # the EXP faults were corrected


def test_allreduce_protect_world2_ipc():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    _check(res, 2)


def test_allreduce_protect_p1_in_process():
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    port = _port()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        from gpu_util import dev, host, sites_to_dev
        rpc = tp.RowParallelCheck(ROWS, N)
        out = []
        for i in range(CALLS):
            parts, bias, bounds, sites = _inputs(i, 1)
            rpc.partial(i).copy_(dev(parts[0]))
            y = torch.empty((ROWS, N), dtype=torch.bfloat16, device="cuda")
            cnt = torch.zeros(ROWS, dtype=torch.int32, device="cuda")
            rpc(i, y, bias=dev(bias), mode=1, bounds=dev(bounds), num_seqs=ROWS, corrected_count=cnt,
                sites=sites_to_dev(sites), n_sites=ROWS, cur_layer=0, cur_step=1)
            torch.cuda.synchronize()
            out.append((host(y).tobytes(), cnt.cpu().numpy().tolist()))
        _check([(0, out, rpc.status())], 1)
        # CUDA-graph replay: the epoch lives in device memory
        g = torch.cuda.CUDAGraph()
        parts, bias, bounds, sites = _inputs(0, 1)
        rpc.partial(0).copy_(dev(parts[0]))
        rpc.partial(1).copy_(dev(parts[0]))
        y = torch.empty((ROWS, N), dtype=torch.bfloat16, device="cuda")
        cnt = torch.zeros(ROWS, dtype=torch.int32, device="cuda")
        bd, bs = dev(bounds), dev(bias)
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            with torch.cuda.graph(g):
                rpc(0, y, bias=bs, mode=1, bounds=bd, num_seqs=ROWS, corrected_count=cnt)
                rpc(1, y, bias=bs, mode=1, bounds=bd, num_seqs=ROWS, corrected_count=cnt)
        for _ in range(3):
            g.replay()
        torch.cuda.synchronize()
        want, wcnt = oracle.allreduce_protect(parts[:1], bias=bias, bounds_=bounds)
        assert np.array_equal(host(y), want) and rpc.status() == 0
        assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), 6 * wcnt)
        assert int(rpc.words[0].item()) == CALLS + 6     # epoch advanced once per call
    finally:
        dist.destroy_process_group()


def test_allreduce_protect_fp16_plain_and_row_map_p1():
    """FP16 (the paper's precision), PLAIN mode (a plain one-shot all-reduce),
    a row -> sequence map with unmapped (-1) rows, no bias; P = 1."""
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    port = _port()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        rows, n = 24, 1024
        rpc = tp.RowParallelCheck(rows, n, dtype=torch.float16)
        rng = np.random.default_rng(4)
        p16 = (rng.standard_normal((rows, n)) * 0.8).astype(np.float16)
        p16.reshape(-1)[::97] = np.float16(np.nan)
        bits = p16.view(np.uint16)
        rpc.partial(0).copy_(torch.from_numpy(bits.view(np.int16).copy()).view(torch.float16).cuda())
        y = torch.empty((rows, n), dtype=torch.float16, device="cuda")
        rpc(0, y, mode=0)                                   # PLAIN: sum (+ no bias), round, no check
        torch.cuda.synchronize()
        want, _ = oracle.allreduce_protect(bits[None], dtype=oracle.DT_FP16)
        got = y.cpu().view(torch.int16).numpy().view(np.uint16)
        assert np.array_equal(got, want)
        S = 3
        r2s = (np.arange(rows) % 4).astype(np.int32) - 1     # rows with -1 are left unchecked
        bnd = np.array([[oracle.f64_to(-0.5, oracle.DT_FP16), oracle.f64_to(0.5, oracle.DT_FP16)],
                        [oracle.f64_to(-1.0, oracle.DT_FP16), oracle.f64_to(0.25, oracle.DT_FP16)],
                        [oracle.f64_to(-0.1, oracle.DT_FP16), oracle.f64_to(2.0, oracle.DT_FP16)]], np.uint16)
        cnt = torch.zeros(S, dtype=torch.int32, device="cuda")
        rpc.partial(1).copy_(rpc.partial(0))
        rpc(1, y, mode=1, bounds=torch.from_numpy(bnd.view(np.int16)).view(torch.float16).cuda(),
            row_to_seq=torch.from_numpy(r2s).cuda(), num_seqs=S, corrected_count=cnt)
        torch.cuda.synchronize()
        want, wcnt = oracle.allreduce_protect(bits[None], bounds_=bnd, row_to_seq=r2s, dtype=oracle.DT_FP16)
        got = y.cpu().view(torch.int16).numpy().view(np.uint16)
        assert np.array_equal(got, want) and np.array_equal(cnt.cpu().numpy().astype(np.uint32), wcnt)
        assert int(wcnt.sum()) > 0 and rpc.status() == 0
    finally:
        dist.destroy_process_group()


def test_allreduce_protect_site_overflow_p1():
    """more than the 64 sites a CTA's list holds, all in one CTA's
    chunk (100 sites on row 0, base_row = 0), are all applied as the oracle's
    R7 applies them."""
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    port = _port()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        from gpu_util import dev, dev_i32, host, sites_to_dev
        rpc = tp.RowParallelCheck(ROWS, N)
        parts, bias, bounds, _ = _inputs(0, 1)
        s = np.zeros(100, oracle.SITE_DTYPE)
        s["step"], s["layer"], s["col"] = 1, 0, (np.arange(100) * 13) % 2048
        s["xor_mask"] = 1 << (np.arange(100) % 16)
        base = np.zeros(100, np.int32)
        rpc.partial(0).copy_(dev(parts[0]))
        y = torch.empty((ROWS, N), dtype=torch.bfloat16, device="cuda")
        cnt = torch.zeros(ROWS, dtype=torch.int32, device="cuda")
        rpc(0, y, bias=dev(bias), mode=1, bounds=dev(bounds), num_seqs=ROWS, corrected_count=cnt,
            sites=sites_to_dev(s), n_sites=100, cur_layer=0, cur_step=1, base_row=dev_i32(base))
        torch.cuda.synchronize()
        want, wcnt = oracle.allreduce_protect(parts[:1], bias=bias, bounds_=bounds, sites=s, cur_layer=0,
                                              cur_step=1, base_row=base)
        plain, _ = oracle.allreduce_protect(parts[:1], bias=bias, bounds_=bounds)
        assert int((want != plain).sum()) > 0
        assert np.array_equal(host(y), want)
        assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), wcnt)
    finally:
        dist.destroy_process_group()


def test_allreduce_protect_p1_in_place():
    """P = 1 with y aliasing this rank's partial and no bias: the kernel writes
    back only the vectors the check (or a fault site) changed, like
    ft2_protect -- the result must still equal the oracle bit for bit, both
    where vectors were rewritten (clipped, faulted) and where they were not."""
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    port = _port()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=0, world_size=1)
    try:
        from gpu_util import dev, host, sites_to_dev
        rpc = tp.RowParallelCheck(ROWS, N)
        for i in range(CALLS):
            parts, _, bounds, sites = _inputs(i, 1)
            y = rpc.partial(i)
            y.copy_(dev(parts[0]))
            cnt = torch.zeros(ROWS, dtype=torch.int32, device="cuda")
            rpc(i, y, mode=1, bounds=dev(bounds), num_seqs=ROWS, corrected_count=cnt,
                sites=sites_to_dev(sites), n_sites=ROWS, cur_layer=0, cur_step=1)
            torch.cuda.synchronize()
            want, wcnt = oracle.allreduce_protect(parts[:1], bounds_=bounds, sites=sites, cur_layer=0, cur_step=1)
            got = host(y)
            assert np.array_equal(got, want), i
            assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), wcnt), i
            changed = (want != parts[0]).reshape(ROWS, N // 8, 8).any(axis=2)
            assert changed.any() and not changed.all()   # both paths ran
        assert rpc.status() == 0
    finally:
        dist.destroy_process_group()
