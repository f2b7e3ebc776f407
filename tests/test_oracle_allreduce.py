"""Pins of the oracle's row-parallel all-reduce + check (SURVEY.md 8(f)
NEXT(2); readings A17, A22): the rank-order fp32 sum is recomputed with numpy
float32 arithmetic and ml_dtypes rounding (an independent implementation of
the same definition), small-integer partials sum exactly, P = 1 reduces to the
single-GPU layer (R5 on RNE(y + bias)), and the check is R5 itself."""
import ml_dtypes
import numpy as np

import ft2_synth
import oracle


def _np_reduce(partials, bias):
    acc = partials[0].view(ml_dtypes.bfloat16).astype(np.float32)
    for t in range(1, partials.shape[0]):
        acc = (acc + partials[t].view(ml_dtypes.bfloat16).astype(np.float32)).astype(np.float32)
    if bias is not None:
        acc = (acc + bias.view(ml_dtypes.bfloat16).astype(np.float32)[None, :]).astype(np.float32)
    return acc.astype(ml_dtypes.bfloat16).view(np.uint16)


def test_rank_order_fp32_sum_matches_numpy():
    P, rows, n = 4, 12, 64
    parts = np.stack([ft2_synth.gen_bf16((rows, n), 40 + t, 3) for t in range(P)])
    bias = ft2_synth.gen_bf16((n,), 50, 3)
    y, _ = oracle.allreduce_protect(parts, bias=bias)
    assert np.array_equal(y, _np_reduce(parts, bias))


def test_small_integers_sum_exactly():
    P, rows, n = 8, 4, 16
    rng = np.random.default_rng(0)
    vals = rng.integers(-20, 21, (P, rows, n)).astype(np.float32)
    parts = vals.astype(ml_dtypes.bfloat16).view(np.uint16)
    y, _ = oracle.allreduce_protect(parts)
    assert np.array_equal(y.view(ml_dtypes.bfloat16).astype(np.float32), vals.sum(0))


def test_p1_is_the_single_gpu_layer_and_check_is_r5():
    rows, n = 16, 128
    p0 = ft2_synth.gen_bf16((rows, n), 60, 4)
    bias = ft2_synth.gen_bf16((n,), 61, 4)
    bounds = np.array([[oracle.f64_to_bf16(-0.4), oracle.f64_to_bf16(0.5)]], np.uint16)
    y, cnt = oracle.allreduce_protect(p0[None], bias=bias, bounds_=bounds)
    want = _np_reduce(p0[None], bias)
    ref_cnt = oracle.protect(want, bounds)
    assert np.array_equal(y, want) and np.array_equal(cnt, ref_cnt) and int(cnt[0]) > 0


def test_faults_then_check():
    P, rows, n = 2, 8, 64
    parts = np.stack([ft2_synth.gen_bf16((rows, n), 70 + t, 5) for t in range(P)])
    sites = oracle.make_sites(3, 0, rows, oracle.FAULT_EXP, [n], n_steps=1, prompt_len=1, step_policy=1)
    bounds = np.array([[oracle.f64_to_bf16(-3.0), oracle.f64_to_bf16(3.0)]] * rows, np.uint16)
    y, cnt = oracle.allreduce_protect(parts, bounds_=bounds, sites=sites, cur_layer=0, cur_step=1)
    want = _np_reduce(parts, None)
    oracle.inject(want, sites, 0, 1)
    ref_cnt = oracle.protect(want, bounds, row_to_seq=np.arange(rows, dtype=np.int32))
    assert np.array_equal(y, want) and np.array_equal(cnt, ref_cnt)
