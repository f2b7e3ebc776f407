"""Pins for the oracle's bounds (R2-R4) and check-and-clip (R5) -- CPU only.

Pinned against:
  * the worked example tests/golden/r2_r5_worked_example.txt (hand-derived);
  * library routines named by the paper: CPU
    ``torch.clamp(torch.nan_to_num(x, nan=0.0), lo, hi)`` and
    ``amin/amax`` over finite values (numeric equality; the +-0 tie edge of
    reading A7 is excluded);
  * the closed form of R3 with scale 2: exactly 2*lo_raw,
    2*hi_raw when lo_raw <= 0 <= hi_raw;
  * invariants of range restriction (BASELINE.json north_star): outputs in
    bounds, in-bound values untouched, idempotent, no NaN/Inf remains, count =
    number of changed elements, monotone;
  * sharding: bounds(concat) == max-combine of per-shard keys.
"""
import os

import ml_dtypes
import numpy as np
import pytest
import torch

import ft2_synth
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "r2_r5_worked_example.txt")


def _gold():
    d = {}
    for line in open(GOLD):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        k, *v = line.split()
        d[k] = [int(x, 16) for x in v] if k not in ("nonfinite", "count") else [int(x) for x in v]
    return d


def _f32(bits):
    return np.asarray(bits, dtype=np.uint16).view(ml_dtypes.bfloat16).astype(np.float32)


def test_worked_example_bounds_and_prefill_correction():
    g = _gold()
    y = np.array(g["prefill"], np.uint16).reshape(2, 4)
    b, k, nf = oracle.bounds(y, scale=2.0, correct_nonfinite=True)
    assert b.tolist() == [g["bounds"]]
    assert k.tolist() == [g["raw_keys"]]
    assert nf.tolist() == g["nonfinite"]
    assert y.reshape(-1).tolist() == g["prefill_after"]


def test_worked_example_decode_clip():
    g = _gold()
    y = np.array(g["decode_in"], np.uint16).reshape(1, 8)
    cnt = oracle.protect(y, np.array([g["bounds"]], np.uint16))
    assert y.reshape(-1).tolist() == g["decode_out"]
    assert cnt.tolist() == g["count"]


def _rand_tensor(rows, n, seed, edges=True):
    y = ft2_synth.gen_bf16((rows, n), tau=7, sigma=seed)
    if edges:
        y = ft2_synth.plant_edge_values(y, stride=53, offset=seed % 17)
    return np.ascontiguousarray(y)


@pytest.mark.parametrize("rows,n,seed", [(1, 8, 1), (3, 24, 2), (17, 40, 3), (64, 128, 4), (5, 1000, 5)])
def test_bounds_vs_torch_amin_amax_of_finite(rows, n, seed):
    y = _rand_tensor(rows, n, seed)
    b, k, nf = oracle.bounds(y.copy(), scale=1.0)
    t = torch.from_numpy(y.view(np.int16)).view(torch.bfloat16).float()
    fin = torch.isfinite(t)
    assert nf[0] == int((~fin).sum())
    lo_raw = oracle.unkey(int(k[0, 0]))
    hi_raw = oracle.unkey(int(k[0, 1]))
    assert _f32([lo_raw])[0] == t[fin].amin().item()
    assert _f32([hi_raw])[0] == t[fin].amax().item()
    # scale = 1.0: the scaled bounds equal the raw ones (exact)
    assert b[0].tolist() == [lo_raw, hi_raw]


def test_bounds_brute_force_tiny_all_sign_mixes():
    rng = np.random.default_rng(3)
    pool = np.array([0x0000, 0x8000, 0x3F80, 0xBF80, 0x0001, 0x8001, 0x7F7F, 0xFF7F, 0x7FC0,
                     0xFFC0, 0x7F80, 0xFF80, 0x4000, 0xC000, 0x3E00, 0xBE00], np.uint16)
    for _ in range(400):
        n = int(rng.integers(1, 7))
        y = rng.choice(pool, size=(1, n)).astype(np.uint16)
        b, k, nf = oracle.bounds(y.copy(), scale=2.0)
        fin = [int(v) for v in y[0] if (v & 0x7F80) != 0x7F80]
        if not fin:
            assert k.tolist() == [[-1, -1]] and b.tolist() == [[0, 0]]   # A9
            continue
        keyed = [(v ^ 0xFFFF) if v & 0x8000 else (v | 0x8000) for v in fin]   # R0 restated
        assert k[0].tolist() == [min(keyed), max(keyed)]
        assert nf[0] == n - len(fin)


def test_scale2_closed_form_and_saturation():
    # R3 with c = 2: lo <= 0 -> 2 lo, hi >= 0 -> 2 hi, exact
    for raw in [0x0000, 0x8000, 0x3F80, 0xBF80, 0x3E9A, 0xC020, 0x0001, 0x8001, 0x7EFF]:
        v = float(_f32([raw])[0])
        if v >= 0:
            assert float(_f32([oracle.scale_bound(raw, 2.0, True)])[0]) == 2 * v
        if v <= 0:
            assert float(_f32([oracle.scale_bound(raw, 2.0, False)])[0]) == 2 * v
    # positive lo / negative hi are divided (sign-aware widening, reading A2)
    assert oracle.scale_bound(0x3F80, 2.0, False) == 0x3F00      # lo 1.0 -> 0.5
    assert oracle.scale_bound(0xBF80, 2.0, True) == 0xBF00       # hi -1 -> -0.5
    # saturation to +-max finite (A8)
    assert oracle.scale_bound(0x7F7F, 2.0, True) == 0x7F7F
    assert oracle.scale_bound(0xFF7F, 2.0, False) == 0xFF7F
    # outward rounding for a non power-of-two factor (A10): 1.25 * 1.0078125
    raw = 0x3F81
    hi = oracle.scale_bound(raw, 1.25, True)
    lo = oracle.scale_bound(raw | 0x8000, 1.25, False)
    exact = 1.25 * float(_f32([raw])[0])
    assert float(_f32([hi])[0]) >= exact and float(_f32([lo])[0]) <= -exact


def test_scaling_commutes_with_min_max():
    # the R3 map is monotone, so scale(min) == min(scale) on every key pair
    rng = np.random.default_rng(4)
    for c in (2.0, 1.25, 3.0):
        for _ in range(300):
            a, b = (int(x) for x in rng.integers(0x0080, 0xFF80, size=2))
            ua, ub = oracle.unkey(a), oracle.unkey(b)
            for is_hi in (False, True):
                sa, sb = oracle.scale_bound(ua, c, is_hi), oracle.scale_bound(ub, c, is_hi)
                if a <= b:
                    assert oracle.key(sa) <= oracle.key(sb)


def test_sharded_bounds_equal_max_combine():
    y = _rand_tensor(12, 96, 9)
    b_full, k_full, nf_full = oracle.bounds(y.copy())
    ks = []
    for part in np.split(y, 4, axis=1):   # column shards (TP column-parallel)
        _, k, _ = oracle.bounds(np.ascontiguousarray(part))
        ks.append(k)
    lo = min(int(k[0, 0]) for k in ks)
    hi = max(int(k[0, 1]) for k in ks)
    assert [lo, hi] == k_full[0].tolist()
    assert oracle.bounds_from_keys(np.array([[lo, hi]])).tolist() == b_full.tolist()


def test_multi_sequence_offsets_and_padding_rows():
    y = _rand_tensor(20, 16, 11)
    so = np.array([2, 5, 5, 12, 19], np.int32)   # rows 0,1 and 19 are padding (A18); seq 1 empty
    b, k, nf = oracle.bounds(y.copy(), seq_offsets=so)
    for s in range(4):
        part = np.ascontiguousarray(y[so[s]:so[s + 1]])
        if part.shape[0] == 0:
            assert k[s].tolist() == [-1, -1] and nf[s] == 0
            continue
        b1, k1, nf1 = oracle.bounds(part)
        assert k[s].tolist() == k1[0].tolist() and b[s].tolist() == b1[0].tolist() and nf[s] == nf1[0]


def test_prefill_correction_changes_only_nonfinite():
    y = _rand_tensor(16, 64, 12)
    y0 = y.copy()
    b, k, nf = oracle.bounds(y, correct_nonfinite=True)
    fin = (y0 & 0x7F80) != 0x7F80
    assert np.array_equal(y[fin], y0[fin])           # R4 invariant (vii)
    assert int((y != y0).sum()) == int((~fin).sum()) == int(nf[0])
    assert not np.any((y & 0x7F80) == 0x7F80)


def _bounds_pair(lo, hi):
    return np.array([[lo, hi]], np.uint16)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_protect_vs_torch_clamp_nan_to_num(seed):
    y = _rand_tensor(32, 256, seed)
    lo, hi = 0xBF00, 0x3F40  # -0.5, 0.75
    out = y.copy()
    cnt = oracle.protect(out, _bounds_pair(lo, hi))
    t = torch.from_numpy(y.view(np.int16)).view(torch.bfloat16)
    ref = torch.clamp(torch.nan_to_num(t, nan=0.0), float(_f32([lo])[0]), float(_f32([hi])[0]))
    ref_bits = ref.view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(out, ref_bits)
    assert cnt[0] == int((out != y).sum())


def test_protect_invariants():
    rng = np.random.default_rng(5)
    for seed in range(6):
        y = _rand_tensor(8, 200, seed + 20)
        kl, kh = sorted(int(x) for x in rng.integers(0x0080, 0xFF80, size=2))
        lo, hi = oracle.unkey(kl), oracle.unkey(kh)
        out = y.copy()
        cnt = oracle.protect(out, _bounds_pair(lo, hi))
        keys = np.where(out & 0x8000, out ^ 0xFFFF, out | 0x8000).astype(np.int64)
        assert np.all((keys >= kl) & (keys <= kh))                    # (i) in bounds
        ykeys = np.where(y & 0x8000, y ^ 0xFFFF, y | 0x8000).astype(np.int64)
        inb = (ykeys >= kl) & (ykeys <= kh) & ((y & 0x7FFF) <= 0x7F80)
        assert np.array_equal(out[inb], y[inb])                        # (ii) untouched
        again = out.copy()
        assert oracle.protect(again, _bounds_pair(lo, hi))[0] == 0     # (iii) idempotent
        assert np.array_equal(again, out)
        assert not np.any((out & 0x7F80) == 0x7F80)                    # (iv) no NaN/Inf
        assert cnt[0] == int((out != y).sum())                         # (v) count
        # (vi) monotone on non-NaN inputs
        nn = (y & 0x7FFF) <= 0x7F80
        order = np.argsort(ykeys[nn], kind="stable")
        assert np.all(np.diff(keys[nn][order]) >= 0)


def test_protect_nan_maps_to_clamped_zero():
    # A5: NaN -> clamp(+0, lo, hi): 0 when lo <= 0 <= hi, else the nearer bound
    for lo, hi, want in [(0xBF80, 0x3F80, 0x0000), (0x3F00, 0x3F80, 0x3F00), (0xBF80, 0xBF00, 0xBF00)]:
        y = np.array([[0x7FC0, 0xFFC1]], np.uint16)
        oracle.protect(y, _bounds_pair(lo, hi))
        assert y.tolist() == [[want, want]]


def test_nan_vulnerable_count_definition():
    # the NaN-vulnerable values are exactly those an exponent-MSB
    # flip turns into NaN, i.e. 1 < |v| < 2 -- checked against numpy decoding and
    # against the flip itself, for bf16 and fp16, per sequence
    import ml_dtypes
    for dt, exp_msb, npdt in ((oracle.DT_BF16, 1 << 14, ml_dtypes.bfloat16), (oracle.DT_FP16, 1 << 14, np.float16)):
        y = _rand_tensor(40, 64, 31)
        y[::3, ::5] = np.array([0x3F90 if dt == 0 else 0x3C10], np.uint16)   # plant values in (1, 2)
        so = [0, 10, 25, 40]
        got = oracle.nan_vulnerable_count(y, so, dtype=dt)
        v = np.abs(y.view(npdt).astype(np.float64))
        want = [int(((v[a:b] > 1) & (v[a:b] < 2)).sum()) for a, b in zip(so[:-1], so[1:])]
        assert got.tolist() == want and sum(want) > 0
        flipped = (y ^ np.uint16(exp_msb)).view(npdt).astype(np.float64)
        nan_after = np.isnan(flipped) & ~np.isnan(y.view(npdt).astype(np.float64))
        assert int(nan_after.sum()) == sum(want)
