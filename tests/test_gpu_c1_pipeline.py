"""Config C1 end to end (BASELINE.json configs[0]): a single critical linear
layer, hidden 768 (OPT-125m-shaped out_proj with bias), 16-token prefill, then
32 decode steps with one seeded single-bit flip per step (step_policy = 1).

Bit-exact part: the GPU bounds / inject / protect kernels
consume the ORACLE's bf16 layer outputs and must reproduce the oracle's
bounds, 32 masks, 32 counts and 32 (col, bit) sites exactly.  The GPU GEMM's
own outputs are checked separately: PLAIN within the GEMM tolerance, and the
fused CHECK+inject epilogue bit-exact against the oracle applied to PLAIN."""
import ml_dtypes
import numpy as np
import pytest
import torch

import ft2_synth
import oracle
from gpu_util import dev, host, sites_to_dev

pytestmark = pytest.mark.gpu

H, T, S = 768, 16, 32


def _inputs():
    w = ft2_synth.gen_bf16((H, H), 1, 1, scale_log2=ft2_synth.weight_scale_log2(H))
    b = ft2_synth.gen_bf16((H,), 3, 1)
    xp = ft2_synth.gen_bf16((T, H), 2, 2)
    xs = [ft2_synth.gen_bf16((1, H), 100 + t, 2) for t in range(1, S + 1)]
    return w, b, xp, xs


def test_c1_pipeline_bit_exact_and_gemm_tolerance():
    import paper_conf_hpdc_sunzmg00y25_b200 as ft2
    w, bias, xp, xs = _inputs()
    # ---- oracle pipeline
    _, yp = oracle.linear_f64(xp, w, bias)
    yp_o = yp.copy()
    rb, rk, rnf = oracle.bounds(yp_o, scale=2.0, correct_nonfinite=True)
    sites = oracle.make_sites(42, 0, S, oracle.FAULT_1BIT, [H], n_steps=S, prompt_len=T, step_policy=1)
    assert sites["step"].tolist() == list(range(1, S + 1))
    base = np.zeros(S, np.int32)
    ys_o, cnt_o, ys_lin = [], [], []
    for t in range(1, S + 1):
        yd_f64, y = oracle.linear_f64(xs[t - 1], w, bias)
        ys_lin.append((yd_f64, y.copy()))
        oracle.inject(y, sites, 0, t, base_row=base)
        c = oracle.protect(y, rb)
        ys_o.append(y)
        cnt_o.append(int(c[0]))
    # ---- GPU kernels on the oracle's layer outputs (bit-exact)
    bd = torch.zeros((1, 2), dtype=torch.bfloat16, device="cuda")
    yp_d = dev(yp)
    ft2.bounds_from_prefill(yp_d, bd, ft2.make_workspace(1), scale=2.0, correct_nonfinite=True)
    assert np.array_equal(host(bd), rb) and np.array_equal(host(yp_d), yp_o)
    sd = ft2.make_fault_sites(42, 0, S, 0, [H], S, T, step_policy=1)
    assert sd.cpu().numpy().tobytes() == sites.tobytes()
    base_d = torch.zeros(S, dtype=torch.int32, device="cuda")
    for t in range(1, S + 1):
        y = dev(ys_lin[t - 1][1])
        cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
        ft2.inject_faults(y, sd, 0, t, base_row=base_d)
        ft2.protect(y, bd, corrected_count=cnt)
        assert np.array_equal(host(y), ys_o[t - 1]), t
        assert int(cnt.item()) == cnt_o[t - 1], t
    # ---- GPU fused GEMM
    wd, bdd = dev(w), dev(bias)
    for t in range(1, S + 1):
        x = dev(xs[t - 1])
        plain = torch.empty((1, H), dtype=torch.bfloat16, device="cuda")
        ft2.protect_fused_gemm(x, wd, plain, bias=bdd, mode=0)
        yd_f64 = ys_lin[t - 1][0]
        g = host(plain).view(ml_dtypes.bfloat16).astype(np.float64)
        tol = 1e-2 * np.maximum(np.abs(yd_f64), 1e-2 * np.sqrt(np.mean(yd_f64 ** 2)))
        assert np.all(np.abs(g - yd_f64) <= tol), t
        fused = torch.empty((1, H), dtype=torch.bfloat16, device="cuda")
        cnt = torch.zeros(1, dtype=torch.int32, device="cuda")
        ft2.protect_fused_gemm(x, wd, fused, bias=bdd, mode=1, bounds=bd, num_seqs=1, corrected_count=cnt,
                               sites=sd, cur_layer=0, cur_step=t, base_row=base_d)
        ref = host(plain).copy()
        oracle.inject(ref, sites, 0, t, base_row=base)
        rc = oracle.protect(ref, rb)
        assert np.array_equal(host(fused), ref) and int(cnt.item()) == int(rc[0]), t
