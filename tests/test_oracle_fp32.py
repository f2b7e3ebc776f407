"""Pins of the oracle's binary32 path (the paper's FP32 study)
against what the mathematics and library routines fix: the 32-bit order key
against numpy's float order, bounds against brute-force finite min/max, the
x2 closed form (L231), outward rounding against exact rationals, the check
against torch.clamp(torch.nan_to_num(x)) (L272), the Fig. 7 / L185 bit-flip
closed forms for binary32, and the SURVEY worked example restated in fp32."""
from fractions import Fraction

import numpy as np
import pytest
import torch

import ft2_synth
import oracle


def f2b(a):
    return np.ascontiguousarray(np.asarray(a, np.float32)).view(np.uint32)


def b2f(a):
    return np.asarray(a, np.uint32).view(np.float32)


def _sample(n, seed):
    rng = np.random.default_rng(seed)
    v = rng.standard_normal(n).astype(np.float32) * np.float32(2.0) ** rng.integers(-20, 20, n).astype(np.float32)
    b = f2b(v)
    specials = [0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x00000001, 0x80000001, 0x7F7FFFFF, 0xFF7FFFFF,
                0x3F800000, 0xBF800000]
    return np.concatenate([b, np.array(specials, np.uint32)])


def test_key32_is_the_float_order():
    b = _sample(4000, 1)
    keys = np.array([oracle.key32(int(x)) for x in b], np.uint64)
    vals = b2f(b).astype(np.float64)
    order_k = np.argsort(keys, kind="stable")
    sv = vals[order_k]
    assert np.all(np.diff(sv) >= 0)                       # key order is value order ...
    sb = b[order_k]
    for i in range(len(sb) - 1):                          # ... with -0 < +0 (A7)
        if sv[i] == sv[i + 1] == 0.0:
            assert not (sb[i] == 0 and sb[i + 1] == 0x80000000)
    for x in b:
        assert oracle.unkey32(oracle.key32(int(x))) == int(x)
    # NaN keys lie outside [key(-Inf), key(+Inf)]
    for nan in (0x7FC00000, 0x7F800001, 0xFFC00000, 0xFFFFFFFF):
        k = oracle.key32(nan)
        assert k < oracle.key32(0xFF800000) or k > oracle.key32(0x7F800000)


def test_bounds32_brute_force_and_x2_closed_form():
    rows, n = 24, 40
    y = (ft2_synth.gen_bf16((rows, n), 4, 9).astype(np.uint32) << 16).reshape(rows, n)  # bf16 -> exact fp32 bits
    y[3, 5] = 0x7FC00000   # NaN
    y[10, 1] = 0xFF800000  # -Inf
    y[20, 7] = 0x7F800000  # +Inf
    so = np.array([0, 8, 8, 24], np.int32)   # one empty sequence
    b, k, have, nf = oracle.bounds32(y.copy(), seq_offsets=so)
    v = b2f(y).astype(np.float64)
    for s in range(3):
        blk = v[so[s]:so[s + 1]]
        fin = blk[np.isfinite(blk)]
        assert nf[s] == blk.size - fin.size
        if fin.size == 0:
            assert have[s] == 0 and b[s].tolist() == [0, 0]
            continue
        lo, hi = fin.min(), fin.max()
        assert lo <= 0 <= hi
        assert b2f(b[s])[0] == 2 * lo and b2f(b[s])[1] == 2 * hi       # exact x2 (L231)
        assert b2f(oracle.unkey32(int(k[s, 0]))) == lo and b2f(oracle.unkey32(int(k[s, 1]))) == hi


def test_bounds32_correction_and_invariants():
    rows, n = 16, 64
    y = f2b(np.random.default_rng(3).standard_normal((rows, n)).astype(np.float32))
    y[0, 0], y[5, 9], y[9, 3] = 0x7FC00000, 0x7F800000, 0xFF800000
    yc = y.copy()
    b, _, _, nf = oracle.bounds32(yc, correct_nonfinite=True)
    assert nf[0] == 3
    changed = yc != y
    assert changed.sum() == 3                             # only non-finite values change (R4)
    assert yc[0, 0] == 0 and yc[5, 9] == b[0, 1] and yc[9, 3] == b[0, 0]


def test_scale_bound32_outward_rounding_exact():
    rng = np.random.default_rng(7)
    for c in (1.25, 1.1, 3.0, 2.0):
        for x in rng.standard_normal(200).astype(np.float32):
            xb = int(f2b(x).reshape(-1)[0])
            for is_hi in (False, True):
                r = oracle.scale_bound32(xb, c, is_hi)
                xf = Fraction(float(x))
                cf = Fraction(float(np.float32(c)))     # the ABI's scale is fp32
                widen = (xf >= 0) if is_hi else (xf <= 0)
                exact = xf * cf if widen else xf / cf
                rv = Fraction(float(b2f(r)))
                if is_hi:
                    assert rv >= exact
                    nxt = Fraction(float(b2f(oracle.unkey32(oracle.key32(r) - 1))))
                    assert nxt < exact or rv == exact
                else:
                    assert rv <= exact
                    nxt = Fraction(float(b2f(oracle.unkey32(oracle.key32(r) + 1))))
                    assert nxt > exact or rv == exact
    assert oracle.scale_bound32(0x7F7FFFFF, 2.0, True) == 0x7F7FFFFF          # saturation (A8)
    assert oracle.scale_bound32(0xFF7FFFFF, 2.0, False) == 0xFF7FFFFF


def test_protect32_matches_torch_clamp_nan_to_num():
    rows, n = 32, 96
    rng = np.random.default_rng(11)
    y = f2b(rng.standard_normal((rows, n)).astype(np.float32) * 3)
    y.reshape(-1)[::53] = 0x7FC00000
    y.reshape(-1)[7::97] = 0x7F800000
    y.reshape(-1)[11::89] = 0xFF800000
    y.reshape(-1)[13::71] = 0xFFC01234     # negative NaN with payload
    bounds = f2b(np.array([[-1.5, 2.25]], np.float32))
    got = y.copy()
    cnt = oracle.protect32(got, bounds)
    want = torch.clamp(torch.nan_to_num(torch.from_numpy(b2f(y).copy()), nan=0.0), -1.5, 2.25).numpy()
    assert np.array_equal(got, f2b(want))
    assert cnt[0] == int((got != y).sum())
    again = got.copy()
    assert oracle.protect32(again, bounds)[0] == 0 and np.array_equal(again, got)   # idempotent
    v = b2f(got)
    assert np.all(np.isfinite(v)) and np.all((v >= -1.5) & (v <= 2.25))
    inb = np.isfinite(b2f(y)) & (b2f(y) >= -1.5) & (b2f(y) <= 2.25)
    assert np.array_equal(got[inb], y[inb])                                         # untouched


def test_fig7_bitflip_closed_forms_fp32():
    """L185 / Fig. 7 for binary32: the top exponent bit (30) of a value in
    (1, 2) gives NaN, of +-1.0 gives +-Inf, of 0.5 gives 2^127, of 2.0 gives 0."""
    sites = np.zeros(1, oracle.SITE_DTYPE)
    sites[0]["xor_mask"] = 1 << 30
    cases = {1.5: None, 1.0: np.inf, -1.0: -np.inf, 0.5: 2.0 ** 127, 2.0: 0.0}
    for x, want in cases.items():
        y = f2b(np.array([[x]], np.float32)).copy()
        oracle.inject32(y, sites, 0, 0)
        got = float(b2f(y)[0, 0])
        if want is None:
            assert np.isnan(got)
        else:
            assert got == want
        oracle.inject32(y, sites, 0, 0)                   # inject o inject = identity
        assert float(b2f(y)[0, 0]) == x


def test_fp32_sites_bit_ranges():
    w = [4096] * 7
    for model, lo, hi, nb in ((0, 0, 32, 1), (1, 0, 32, 2), (2, 23, 31, 1)):
        s = oracle.make_sites(5, 0, 4000, model, w, 32, 16, dtype=oracle.DT_FP32)
        masks = s["xor_mask"].astype(np.uint64)
        pc = np.array([bin(int(m)).count("1") for m in masks])
        assert np.all(pc == nb)
        bits = set()
        for m in masks:
            bits |= {i for i in range(32) if (int(m) >> i) & 1}
        assert min(bits) >= lo and max(bits) < hi
        assert len(bits) == hi - lo                       # every allowed position is drawn


def test_worked_example_in_fp32():
    """SURVEY §8(c)'s R2-R5 worked example (tests/golden/r2_r5_worked_example.txt)
    restated in binary32: every value is exactly representable, so the
    bounds, corrections and count are the same numbers."""
    pre = f2b(np.array([[0.5, -0.75, np.nan, 1.25], [-0.0, 0.0, np.inf, -2.5]], np.float32)).copy()
    b, _, _, nf = oracle.bounds32(pre, correct_nonfinite=True)
    assert b2f(b[0]).tolist() == [-5.0, 2.5] and nf[0] == 2
    assert b2f(pre).tolist() == [[0.5, -0.75, 0.0, 1.25], [-0.0, 0.0, 2.5, -2.5]]
    assert pre[1, 0] == 0x80000000                       # -0 stays -0
    dec = f2b(np.array([[0.30078125, -6, 3, np.nan, -np.inf, 2.5, -5, 65536]], np.float32)).copy()
    cnt = oracle.protect32(dec, b)
    assert b2f(dec).tolist() == [[0.30078125, -5.0, 2.5, 0.0, -5.0, 2.5, -5.0, 2.5]] and cnt[0] == 5
