"""Pins for the reference linear layer (R8) -- CPU.

Pinned against: exact integer arithmetic (small-integer inputs make every
product and sum exact, so the result is known in closed form), the fp64
numpy matmul as an independent library primitive on random inputs, and the
composition order GEMM -> bias -> bf16 -> inject -> check (reading A19/A20).
"""
import ml_dtypes
import numpy as np

import ft2_synth
import oracle


def _bits(a):
    return np.asarray(a, np.float32).astype(ml_dtypes.bfloat16).view(np.uint16)


def _f64(b):
    return np.asarray(b, np.uint16).view(ml_dtypes.bfloat16).astype(np.float64)


def test_linear_exact_on_small_integers():
    rng = np.random.default_rng(0)
    x = rng.integers(-3, 4, size=(5, 33)).astype(np.float32)
    w = rng.integers(-3, 4, size=(7, 33)).astype(np.float32)
    b = rng.integers(-5, 6, size=7).astype(np.float32)
    yd, yb = oracle.linear_f64(_bits(x), _bits(w), _bits(b))
    want = x.astype(np.int64) @ w.T.astype(np.int64) + b.astype(np.int64)
    assert np.array_equal(yd, want.astype(np.float64))
    assert np.array_equal(_f64(yb), want.astype(np.float64))   # |y| < 256: exact in bf16


def test_linear_matches_numpy_fp64_on_synthetic_inputs():
    M, N, K = 4, 48, 200
    x = ft2_synth.gen_bf16((M, K), 1, 2)
    w = ft2_synth.gen_bf16((N, K), 2, 1, scale_log2=ft2_synth.weight_scale_log2(K))
    bias = ft2_synth.gen_bf16((N,), 3, 1)
    yd, yb = oracle.linear_f64(x, w, bias)
    ref = _f64(x) @ _f64(w).T + _f64(bias)
    assert np.allclose(yd, ref, rtol=1e-12, atol=1e-12)
    # one rounding to bf16: relative error at most half an ulp (2^-8 of the value)
    assert np.max(np.abs(_f64(yb) - ref) / np.maximum(np.abs(ref), 1e-30)) <= 2 ** -8


def test_protected_linear_order_inject_then_check():
    M, N, K = 2, 16, 32
    x = ft2_synth.gen_bf16((M, K), 4, 2)
    w = ft2_synth.gen_bf16((N, K), 5, 1, scale_log2=-3)
    _, yb = oracle.linear_f64(x, w)
    s = np.zeros(1, oracle.SITE_DTYPE)
    s["step"], s["layer"], s["col"], s["xor_mask"] = 5, 3, 7, 1 << 14
    bnd = np.array([[0xC000, 0x4000]], np.uint16)   # [-2, 2]
    y, cnt = oracle.protected_linear(x, w, None, bnd, row_to_seq=np.zeros(M, np.int32), sites=s,
                                     cur_layer=3, cur_step=5, base_row=np.array([1], np.int32))
    ref = yb.copy()
    ref[1, 7] ^= 1 << 14                        # R7 on the bf16-rounded value
    c = oracle.protect(ref, bnd, row_to_seq=np.zeros(M, np.int32))
    assert np.array_equal(y, ref) and cnt.tolist() == c.tolist()
    assert cnt[0] >= 1                           # the flipped value was out of [-2, 2] or NaN


def test_oracle_results_do_not_depend_on_thread_count():
    """The oracle's OpenMP loops run over independent outputs (each computed by
    one thread in the stated order): 1 thread and all threads give identical
    bits, counts and keys."""
    import ft2_synth
    x = ft2_synth.gen_bf16((7, 136), 1, 2)
    w = ft2_synth.gen_bf16((200, 136), 2, 2, scale_log2=-4)
    b = ft2_synth.gen_bf16((200,), 3, 2)
    y = ft2_synth.plant_edge_values(ft2_synth.gen_bf16((64, 264), 4, 2))
    so = np.array([0, 5, 5, 30, 64], np.int32)
    out = []
    for n in (1, 0):
        oracle.set_threads(n)
        d, lb = oracle.linear_f64(x, w, b)
        yy = y.copy()
        bnd, keys, nf = oracle.bounds(yy, seq_offsets=so, correct_nonfinite=True)
        z = y.copy()
        cnt = oracle.protect(z, bnd, row_to_seq=np.repeat(np.arange(4, dtype=np.int32), [5, 0, 25, 34]))
        out.append((d.tobytes(), lb.tobytes(), yy.tobytes(), bnd.tobytes(), keys.tobytes(), nf.tobytes(),
                    z.tobytes(), cnt.tobytes()))
    oracle.set_threads(0)
    assert out[0] == out[1]
