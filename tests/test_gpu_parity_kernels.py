"""GPU parity of the bounds, check-and-clip, fault-site and injection kernels
against the CPU oracle -- bit-exact (BASELINE.json north_star: "bit-exact for
bounds, clip masks, corrected counts and injected bit positions").

Every call goes through the C ABI (libft2.so via the ctypes binding).
"""
import numpy as np
import pytest
import torch

import ft2_synth
import oracle
from gpu_util import dev, dev_i32, host, sites_to_dev, sites_to_host

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ft2():
    import paper_conf_hpdc_sunzmg00y25_b200 as m
    return m


def _tensor(rows, n, seed, edges=True, tau=3):
    y = ft2_synth.gen_bf16((rows, n), tau=tau, sigma=seed)
    if edges:
        y = ft2_synth.plant_edge_values(y, stride=211, offset=seed % 37)
    return np.ascontiguousarray(y)


def _rand_bounds(S, seed):
    rng = np.random.default_rng(seed)
    out = np.zeros((S, 2), np.uint16)
    for s in range(S):
        # bounds drawn around the bulk of the data so that some values are clipped
        lo = -abs(rng.normal(0.6, 0.3)) - 0.05
        hi = abs(rng.normal(0.6, 0.3)) + 0.05
        out[s] = [oracle.f64_to_bf16(lo), oracle.f64_to_bf16(hi)]
    return out


# ----------------------------------------------------------------- protect --
# (1600, 8200): 13.1M elements, more than two full waves of the grid-stride
# loop (148 SMs x 5 CTAs x 256 threads x 4 vectors x 8 elements) plus a ragged tail
PROTECT_SHAPES = [(1, 8), (1, 768), (3, 24), (17, 40), (7, 1000), (32, 2048), (32, 11008), (129, 4096),
                  (512, 4104), (1600, 8200)]


@pytest.mark.parametrize("rows,n", PROTECT_SHAPES)
@pytest.mark.parametrize("mapping", ["single", "per_row", "array"])
def test_protect_bit_exact(ft2, rows, n, mapping):
    y = _tensor(rows, n, seed=rows * 7 + n)
    if mapping == "single":
        S, r2s = 1, None
    elif mapping == "per_row":
        S, r2s = rows, None
    else:
        S = 3
        r2s = (np.arange(rows) % 4).astype(np.int32) - 1   # -1 rows are left alone
    b = _rand_bounds(S, rows + n)
    ref = y.copy()
    ref_cnt = oracle.protect(ref, b, row_to_seq=r2s if r2s is not None else
                             (None if S == 1 else np.arange(rows, dtype=np.int32)))
    yd = dev(y)
    cnt = torch.zeros(S, dtype=torch.int32, device="cuda")
    ft2.protect(yd, dev(b), row_to_seq=None if r2s is None else dev_i32(r2s), num_seqs=S, corrected_count=cnt)
    torch.cuda.synchronize()
    assert np.array_equal(host(yd), ref)
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), ref_cnt)


def test_protect_strided_view_and_idempotence(ft2):
    y = _tensor(64, 3 * 512, seed=5)
    b = _rand_bounds(1, 9)
    full = dev(y)
    view = full[:, 512:1024]     # the "V of a fused QKV" slice, ld = 1536
    ref = np.ascontiguousarray(y[:, 512:1024])
    rc = oracle.protect(ref, b)
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect(view, dev(b), corrected_count=cnt)
    out = host(full)
    assert np.array_equal(out[:, 512:1024], ref) and int(cnt.item()) == int(rc[0])
    assert np.array_equal(out[:, :512], y[:, :512]) and np.array_equal(out[:, 1024:], y[:, 1024:])
    ft2.protect(view, dev(b), corrected_count=cnt)   # second pass changes nothing
    assert np.array_equal(host(full), out) and int(cnt.item()) == int(rc[0])


def test_protect_worked_example(ft2):
    y = np.array([[0x3E9A, 0xC0C0, 0x4040, 0x7FC0, 0xFF80, 0x4020, 0xC0A0, 0x4780]], np.uint16)
    yd = dev(y)
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect(yd, dev(np.array([[0xC0A0, 0x4020]], np.uint16)), corrected_count=cnt)
    assert host(yd).tolist() == [[0x3E9A, 0xC0A0, 0x4020, 0x0000, 0xC0A0, 0x4020, 0xC0A0, 0x4020]]
    assert cnt.item() == 5


# ------------------------------------------------------------------ bounds --
def _gpu_bounds(ft2, y, so, scale=2.0, correct=False, finalize=True):
    S = 1 if so is None else len(so) - 1
    yd = dev(y)
    b = torch.zeros((S, 2), dtype=torch.bfloat16, device="cuda")
    k = torch.zeros((S, 2), dtype=torch.int32, device="cuda")
    nf = torch.zeros(S, dtype=torch.int32, device="cuda")
    ws = ft2.make_workspace(S)
    ft2.bounds_from_prefill(yd, b if finalize else None, ws, seq_offsets=None if so is None else dev_i32(so),
                            num_seqs=S, scale=scale, finalize=finalize, correct_nonfinite=correct, keys_out=k,
                            nonfinite_count=nf)
    torch.cuda.synchronize()
    assert int(ws.abs().sum().item()) == 0, "workspace must be left zero-filled"
    return host(yd), host(b), k.cpu().numpy(), nf.cpu().numpy().astype(np.uint32)


def _oracle_keys_encoded(k):
    # oracle raw keys (min, max) -> ABI keys_out encoding (0xFFFF - min, max), -1 stays -1
    out = k.copy()
    out[:, 0] = np.where(k[:, 0] >= 0, 0xFFFF - k[:, 0], -1)
    return out


BOUNDS_CASES = [
    ((2, 8), None), ((16, 768), None), ((3, 24), [0, 1, 3]), ((17, 40), [2, 5, 5, 12, 16]),
    ((128, 2048), None), ((512, 4096), list(range(0, 513, 16))), ((100, 11008), [0, 37, 37, 100]),
    ((4096, 2048), list(range(0, 4097, 128))), ((33, 1000), [1, 2, 3, 30]),
]


@pytest.mark.parametrize("shape,so", BOUNDS_CASES)
@pytest.mark.parametrize("correct", [False, True])
def test_bounds_bit_exact(ft2, shape, so, correct):
    y = _tensor(*shape, seed=shape[0] + shape[1])
    ref = y.copy()
    rb, rk, rnf = oracle.bounds(ref, seq_offsets=so, correct_nonfinite=correct)
    out, b, k, nf = _gpu_bounds(ft2, y, so, correct=correct)
    assert np.array_equal(b, rb)
    assert np.array_equal(k, _oracle_keys_encoded(rk))
    assert np.array_equal(nf, rnf)
    assert np.array_equal(out, ref)   # correction (or untouched input)


@pytest.mark.parametrize("shape,so", BOUNDS_CASES)
def test_nan_vulnerable_count_bit_exact(ft2, shape, so):
    """NaN-vulnerable values (Fig. 7), counted in the bounds sweep."""
    y = _tensor(*shape, seed=shape[0] * 3 + shape[1])
    y.reshape(-1)[5::97] = 0x3FC0          # 1.5: inside (1, 2)
    y.reshape(-1)[11::89] = 0xBF80         # -1.0: boundary, not counted
    want = oracle.nan_vulnerable_count(y, seq_offsets=so)
    ref = y.copy()
    rb, _, _ = oracle.bounds(ref, seq_offsets=so, correct_nonfinite=True)
    S = 1 if so is None else len(so) - 1
    yd = dev(y)
    b = torch.zeros((S, 2), dtype=torch.bfloat16, device="cuda")
    nv = torch.full((S,), -1, dtype=torch.int32, device="cuda")
    ws = ft2.make_workspace(S)
    ft2.bounds_from_prefill(yd, b, ws, seq_offsets=None if so is None else dev_i32(so), num_seqs=S,
                            correct_nonfinite=True, nan_vulnerable_count=nv)
    torch.cuda.synchronize()
    assert np.array_equal(nv.cpu().numpy().astype(np.uint32), want) and int(want.sum()) > 0
    assert np.array_equal(host(b), rb) and np.array_equal(host(yd), ref)
    assert int(ws.abs().sum().item()) == 0


@pytest.mark.parametrize("scale", [1.0, 1.25, 2.0, 3.0])
def test_bounds_scales(ft2, scale):
    y = _tensor(64, 512, seed=17)
    rb, rk, _ = oracle.bounds(y.copy(), scale=scale)
    _, b, k, _ = _gpu_bounds(ft2, y, None, scale=scale)
    assert np.array_equal(b, rb)


def test_bounds_keys_only_then_finalize(ft2):
    y = _tensor(40, 256, seed=4)
    so = [0, 10, 30, 40]
    rb, rk, _ = oracle.bounds(y.copy(), seq_offsets=so)
    _, _, k, _ = _gpu_bounds(ft2, y, so, finalize=False)
    assert np.array_equal(k, _oracle_keys_encoded(rk))
    b = torch.zeros((3, 2), dtype=torch.bfloat16, device="cuda")
    ft2.bounds_finalize(torch.as_tensor(k).cuda(), b)
    assert np.array_equal(host(b), rb)


def test_bounds_degenerate_sequences(ft2):
    # all-NaN sequence (A9), all-negative, all-positive, single element, many Inf (patch overflow)
    y = _tensor(6, 4096, seed=8, edges=False)
    y[0, :] = 0x7FC0
    y[1, :] = np.abs(y[1, :].view(np.int16)).view(np.uint16) | 0x8000          # all negative
    y[2, :] = y[2, :] & 0x7FFF                                                   # all positive
    y[3, ::2] = 0x7F80                                                           # 2048 +Inf
    y[4, :] = 0xFF80                                                             # 4096 -Inf -> overflow path
    so = [0, 1, 2, 3, 4, 5, 6]
    ref = y.copy()
    rb, rk, rnf = oracle.bounds(ref, seq_offsets=so, correct_nonfinite=True)
    out, b, k, nf = _gpu_bounds(ft2, y, so, correct=True)
    assert rb[0].tolist() == [0, 0] and rk[0].tolist() == [-1, -1]
    assert np.array_equal(b, rb) and np.array_equal(nf, rnf) and np.array_equal(out, ref)


def test_bounds_worked_example(ft2):
    y = np.array([[0x3F00, 0xBF40, 0x7FC0, 0x3FA0, 0x8000, 0x0000, 0x7F80, 0xC020]], np.uint16).reshape(1, 8)
    out, b, k, nf = _gpu_bounds(ft2, y, None, correct=True)
    assert b.tolist() == [[0xC0A0, 0x4020]] and nf.tolist() == [2]
    assert out.reshape(-1).tolist() == [0x3F00, 0xBF40, 0x0000, 0x3FA0, 0x8000, 0x0000, 0x4020, 0xC020]


def test_bounds_and_protect_full_size(ft2):
    """BASELINE full size: Llama-2-7B prefill up_proj, 32 x 2048 tokens: [65536, 11008] = 1.44 GB."""
    rows, n = 65536, 11008
    yd = ft2_synth.gen_bf16_torch((rows, n), tau=11, sigma=5, device="cuda")
    yh = host(yd)
    rb, rk, rnf = oracle.bounds(yh, seq_offsets=None)
    b = torch.zeros((1, 2), dtype=torch.bfloat16, device="cuda")
    k = torch.zeros((1, 2), dtype=torch.int32, device="cuda")
    ws = ft2.make_workspace(1)
    ft2.bounds_from_prefill(yd, b, ws, keys_out=k)
    assert np.array_equal(host(b), rb) and np.array_equal(k.cpu().numpy(), _oracle_keys_encoded(rk))
    # 32 sequences of 2048 tokens
    so = list(range(0, rows + 1, 2048))
    rb32, _, _ = oracle.bounds(yh, seq_offsets=so)
    b32 = torch.zeros((32, 2), dtype=torch.bfloat16, device="cuda")
    ft2.bounds_from_prefill(yd, b32, ft2.make_workspace(32), seq_offsets=dev_i32(so))
    assert np.array_equal(host(b32), rb32)
    # check-and-clip at full size against tighter bounds
    tb = np.array([[oracle.f64_to_bf16(-0.5), oracle.f64_to_bf16(0.5)]], np.uint16)
    ref = yh.copy()
    rc = oracle.protect(ref, tb)
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect(yd, dev(tb), corrected_count=cnt)
    assert int(cnt.item()) == int(rc[0])
    assert np.array_equal(host(yd), ref)


# ------------------------------------------------------------ fault sites --
LLAMA7B = [4096, 4096, 4096, 4096, 11008, 11008, 4096] * 32
OPT13B = [2048, 2048, 2048, 2048, 8192, 2048] * 24


@pytest.mark.parametrize("model", [0, 1, 2])
@pytest.mark.parametrize("geom", ["llama7b", "opt13b_neuron", "c1_per_step"])
def test_fault_sites_bit_exact(ft2, model, geom):
    if geom == "llama7b":
        w, S, T, lu, sp, n, t0 = LLAMA7B, 32, 16, True, 0, 100000, 0
    elif geom == "opt13b_neuron":
        w, S, T, lu, sp, n, t0 = OPT13B, 60, 128, False, 0, 20000, 12345
    else:
        w, S, T, lu, sp, n, t0 = [768], 32, 16, True, 1, 32, 0
    ref = oracle.make_sites(42 + model, t0, n, model, w, S, T, layer_uniform=lu, step_policy=sp)
    got = ft2.make_fault_sites(42 + model, t0, n, model, w, S, T, layer_uniform=lu, step_policy=sp)
    torch.cuda.synchronize()
    assert got.cpu().numpy().tobytes() == ref.tobytes()


def test_inject_bit_exact(ft2):
    sites = oracle.make_sites(7, 0, 256, 2, [512] * 4, n_steps=3, prompt_len=8)
    y = _tensor(256, 512, seed=3, edges=False)
    sd = sites_to_dev(sites)
    for layer in range(4):
        for step in range(1, 4):
            ref = y.copy()
            oracle.inject(ref, sites, layer, step)
            yd = dev(y)
            ft2.inject_faults(yd, sd, layer, step)
            assert np.array_equal(host(yd), ref)
    # prefill: base_row = seq_offsets, token offsets inside each sequence
    y2 = _tensor(256 * 8, 512, seed=4, edges=False)
    base = np.arange(256, dtype=np.int32) * 8
    for layer in range(4):
        ref = y2.copy()
        oracle.inject(ref, sites, layer, 0, base_row=base)
        yd = dev(y2)
        ft2.inject_faults(yd, sd, layer, 0, base_row=dev_i32(base))
        assert np.array_equal(host(yd), ref)


def test_tp_sharded_bounds_equal_unsharded(ft2):
    """Column shards -> keys (finalize=0) -> MAX combine -> finalize == unsharded bounds (bit-exact)."""
    rows, n, world = 256, 4096, 4
    y = _tensor(rows, n, seed=21)
    so = [0, 64, 64, 200, 256]
    rb, rk, _ = oracle.bounds(y.copy(), seq_offsets=so)
    keys = []
    for r in range(world):
        shard = np.ascontiguousarray(y[:, r * n // world:(r + 1) * n // world])
        _, _, k, _ = _gpu_bounds(ft2, shard, so, finalize=False)
        keys.append(torch.as_tensor(k))
    comb = torch.stack(keys).amax(0).contiguous()
    assert np.array_equal(comb.numpy(), _oracle_keys_encoded(rk))
    b = torch.zeros((4, 2), dtype=torch.bfloat16, device="cuda")
    ft2.bounds_finalize(comb.cuda(), b)
    assert np.array_equal(host(b), rb)


def test_tp_bounds_nccl_world1(ft2):
    """The product TP path (kernel keys -> NCCL MAX all-reduce -> finalize) on a 1-rank NCCL group."""
    import socket
    import torch.distributed as dist
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    if not dist.is_initialized():
        s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
        dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    y = _tensor(128, 1024, seed=22)
    so = [0, 32, 128]
    rb, _, _ = oracle.bounds(y.copy(), seq_offsets=so)
    b = torch.zeros((2, 2), dtype=torch.bfloat16, device="cuda")
    tp.tp_bounds_from_prefill(dev(y), b, ft2.make_workspace(2), seq_offsets=dev_i32(so), num_seqs=2)
    assert np.array_equal(host(b), rb)
    dist.destroy_process_group()
