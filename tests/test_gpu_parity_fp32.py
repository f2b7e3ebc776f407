"""GPU parity of the binary32 path (the paper's FP32 study):
bounds (+ non-finite correction, raw keys, counts), check-and-clip, injection
and the tensor-parallel keys/finalize, bit-exact against the oracle's fp32
functions on the same seeded inputs."""
import numpy as np
import pytest
import torch

import oracle
from gpu_util import dev_i32

pytestmark = pytest.mark.gpu

INT32_MIN = -(1 << 31)


@pytest.fixture(scope="module")
def ft2():
    import paper_conf_hpdc_sunzmg00y25_b200 as m
    return m


def dev32(a):
    a = np.ascontiguousarray(a, np.uint32)
    return torch.from_numpy(a.view(np.int32).copy()).view(torch.float32).cuda()


def host32(t):
    return t.detach().contiguous().cpu().view(torch.int32).numpy().view(np.uint32)


def _tensor32(rows, n, seed, edges=True):
    """Seeded fp32 activations: normal bulk, rare x32..x256 outliers (L261),
    and planted NaN (both signs, payloads), +-Inf, +-0, subnormals, +-FLT_MAX."""
    rng = np.random.default_rng(seed)
    v = (rng.standard_normal((rows, n)) * 0.3).astype(np.float32)
    out = rng.random((rows, n)) < 2.0 ** -10
    v[out] *= np.float32(2.0) ** rng.integers(5, 9, out.sum()).astype(np.float32)
    b = v.view(np.uint32).copy()
    if edges:
        flat = b.reshape(-1)
        specials = np.array([0x7FC00000, 0xFFC00001, 0x7F800001, 0x7F800000, 0xFF800000, 0x00000000, 0x80000000,
                             0x00000007, 0x80400000, 0x7F7FFFFF, 0xFF7FFFFF], np.uint32)
        idx = np.arange(seed % 29, flat.size, 1009)
        flat[idx] = specials[np.arange(idx.size) % specials.size]
    return b


def _gpu_bounds32(ft2, y, so, scale=2.0, correct=False):
    S = 1 if so is None else len(so) - 1
    yd = dev32(y)
    b = torch.zeros((S, 2), dtype=torch.float32, device="cuda")
    k = torch.zeros((S, 2), dtype=torch.int32, device="cuda")
    nf = torch.zeros(S, dtype=torch.int32, device="cuda")
    ws = ft2.make_workspace(S)
    ft2.bounds_from_prefill(yd, b, ws, seq_offsets=None if so is None else dev_i32(so), num_seqs=S, scale=scale,
                            correct_nonfinite=correct, keys_out=k, nonfinite_count=nf)
    torch.cuda.synchronize()
    assert int(ws.abs().sum().item()) == 0, "workspace must be left zero-filled"
    return host32(yd), host32(b), k.cpu().numpy(), nf.cpu().numpy().astype(np.uint32)


def _enc(raw, have):
    """oracle raw 32-bit keys -> the ABI's MAX-combinable int32 encoding."""
    lo = np.where(have != 0, (~raw[:, 0].astype(np.uint32)) ^ np.uint32(0x80000000), np.uint32(0x80000000))
    hi = np.where(have != 0, raw[:, 1].astype(np.uint32) ^ np.uint32(0x80000000), np.uint32(0x80000000))
    return np.stack([lo, hi], 1).view(np.int32)


BOUNDS_CASES = [((1, 4), None), ((16, 768), None), ((37, 1000), [0, 5, 5, 20, 37]),
                ((128, 4096), list(range(0, 129, 16))), ((600, 2048), [3, 100, 400, 590]),
                ((4096, 4096), list(range(0, 4097, 128)))]


@pytest.mark.parametrize("shape,so", BOUNDS_CASES)
@pytest.mark.parametrize("correct", [False, True])
def test_bounds32_bit_exact(ft2, shape, so, correct):
    rows, n = shape
    y = _tensor32(rows, n, seed=rows + n)
    so_np = None if so is None else np.array(so, np.int32)
    ref = y.copy()
    rb, rk, rh, rnf = oracle.bounds32(ref, seq_offsets=so_np, correct_nonfinite=correct)
    gy, gb, gk, gnf = _gpu_bounds32(ft2, y, so_np, correct=correct)
    assert np.array_equal(gb, rb)
    assert np.array_equal(gk, _enc(rk, rh))
    assert np.array_equal(gnf, rnf)
    assert np.array_equal(gy, ref if correct else y)


def test_bounds32_scale_125_and_all_nonfinite(ft2):
    y = _tensor32(64, 512, seed=3)
    ref = y.copy()
    rb, _, _, _ = oracle.bounds32(ref, scale=1.25)
    _, gb, _, _ = _gpu_bounds32(ft2, y, None, scale=1.25)
    assert np.array_equal(gb, rb)
    bad = np.full((4, 8), 0x7FC00000, np.uint32)                     # A9: no finite value
    bad[1, 3] = 0xFF800000
    rb, rk, rh, rnf = oracle.bounds32(bad.copy(), correct_nonfinite=True)
    gy, gb, gk, gnf = _gpu_bounds32(ft2, bad, None, correct=True)
    assert rh[0] == 0 and gb.tolist() == rb.tolist() == [[0, 0]] and gk.tolist() == [[INT32_MIN, INT32_MIN]]
    assert int(gnf[0]) == 32 and np.all(gy == 0)


def test_bounds32_patch_list_overflow(ft2):
    """More non-finite values than the patch list holds: the last CTA sweeps."""
    y = _tensor32(256, 2048, seed=8, edges=False)
    y.reshape(-1)[::97] = 0x7FC00000
    so = np.array([0, 100, 256], np.int32)
    ref = y.copy()
    rb, _, _, rnf = oracle.bounds32(ref, seq_offsets=so, correct_nonfinite=True)
    gy, gb, _, gnf = _gpu_bounds32(ft2, y, so, correct=True)
    assert int(rnf.sum()) > 4096
    assert np.array_equal(gb, rb) and np.array_equal(gnf, rnf) and np.array_equal(gy, ref)


# (1500, 4100): 6.15M elements, more than two waves of the 740-CTA grid
# (4 vectors x 4 values per thread per pass) plus a ragged tail
@pytest.mark.parametrize("rows,n", [(1, 4), (3, 20), (32, 2048), (33, 11008), (512, 4100), (1500, 4100)])
@pytest.mark.parametrize("mapping", ["single", "per_row", "array"])
def test_protect32_bit_exact(ft2, rows, n, mapping):
    y = _tensor32(rows, n, seed=rows * 3 + n)
    rng = np.random.default_rng(rows + n)
    if mapping == "single":
        S, r2s = 1, None
    elif mapping == "per_row":
        S, r2s = rows, None
    else:
        S, r2s = 3, (np.arange(rows) % 4).astype(np.int32) - 1
    b = np.stack([-np.abs(rng.normal(0.6, 0.3, S)) - 0.05, np.abs(rng.normal(0.6, 0.3, S)) + 0.05], 1)
    b = b.astype(np.float32).view(np.uint32)
    ref = y.copy()
    rc = oracle.protect32(ref, b, row_to_seq=r2s if r2s is not None else
                          (None if S == 1 else np.arange(rows, dtype=np.int32)))
    yd = dev32(y)
    cnt = torch.zeros(S, dtype=torch.int32, device="cuda")
    ft2.protect(yd, dev32(b), row_to_seq=None if r2s is None else dev_i32(r2s), num_seqs=S, corrected_count=cnt)
    torch.cuda.synchronize()
    assert np.array_equal(host32(yd), ref)
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), rc)


def test_protect32_strided_view(ft2):
    y = _tensor32(64, 3 * 256, seed=5)
    b = np.array([[-0.5, 0.75]], np.float32).view(np.uint32)
    full = dev32(y)
    ref = np.ascontiguousarray(y[:, 256:512])
    rc = oracle.protect32(ref, b)
    cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
    ft2.protect(full[:, 256:512], dev32(b), corrected_count=cnt)
    out = host32(full)
    assert np.array_equal(out[:, 256:512], ref) and int(cnt.item()) == int(rc[0])
    assert np.array_equal(out[:, :256], y[:, :256]) and np.array_equal(out[:, 512:], y[:, 512:])


def test_inject32_bit_exact(ft2):
    w = [1024, 4096, 1024]
    for model in (0, 1, 2):
        sites = oracle.make_sites(17, 0, 64, model, w, n_steps=4, prompt_len=8, dtype=oracle.DT_FP32)
        sd = ft2.make_fault_sites(17, 0, 64, model, w, 4, 8, dtype=2)
        assert sd.cpu().numpy().tobytes() == sites.tobytes()
        for step in range(0, 5):
            for layer in range(3):
                y = _tensor32(64 * (8 if step == 0 else 1), w[layer], seed=step * 7 + layer, edges=False)
                base = np.arange(64, dtype=np.int32) * (8 if step == 0 else 1)
                ref = oracle.inject32(y.copy(), sites, layer, step, base_row=base)
                yd = dev32(y)
                ft2.inject_faults(yd, sd, layer, step, base_row=dev_i32(base))
                assert np.array_equal(host32(yd), ref), (model, step, layer)


@pytest.mark.parametrize("P", [2, 8])
def test_tp_keys_fp32_combine(ft2, P):
    from paper_conf_hpdc_sunzmg00y25_b200 import tp
    rows, n = 96, 5120
    y = _tensor32(rows, n, seed=P)
    so = np.array([0, 16, 16, 50, 96], np.int32)
    rb, rk, rh, _ = oracle.bounds32(y.copy(), seq_offsets=so)
    yd, sod = dev32(y), dev_i32(so)
    comb = None
    for r in range(P):
        b0, e0 = tp.column_shard(n, P, r)
        k = torch.empty((4, 2), dtype=torch.int32, device="cuda")
        ft2.bounds_from_prefill(yd[:, b0:e0], None, ft2.make_workspace(4), seq_offsets=sod, num_seqs=4,
                                finalize=False, keys_out=k)
        comb = k if comb is None else torch.maximum(comb, k)
    assert np.array_equal(comb.cpu().numpy(), _enc(rk, rh))
    bnd = torch.zeros((4, 2), dtype=torch.float32, device="cuda")
    ft2.bounds_finalize(comb, bnd)
    assert np.array_equal(host32(bnd), rb)


def test_fused_gemm_fp32_unsupported(ft2):
    x = torch.zeros((4, 64), dtype=torch.float32, device="cuda")
    w = torch.zeros((64, 64), dtype=torch.float32, device="cuda")
    y = torch.zeros((4, 64), dtype=torch.float32, device="cuda")
    with pytest.raises(Exception, match="UNSUPPORTED"):
        ft2.protect_fused_gemm(x, w, y, mode=0)
