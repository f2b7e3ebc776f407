"""The shared input generator (ft2_synth) -- CPU.

Golden values: SURVEY.md 8(d) (seed 2, tensor 0, i = 0..7) and the Philox
known-answer vectors; host (numpy) and torch implementations must agree.
"""
import numpy as np
import torch

import ft2_synth


def test_golden_values():
    g = ft2_synth.gen_bf16((8,), tau=0, sigma=2)
    assert g.tolist() == [0x3F1F, 0xBE97, 0xBEE8, 0xBE82, 0x3EAE, 0x3ED5, 0xBE9A, 0xBE41]


def test_numpy_and_torch_agree():
    for shape, tau, sigma, sl in [((1000,), 0, 2, 0), ((37, 129), 5, 1 << 40, -6), ((3, 5), 9, 7, 3)]:
        a = ft2_synth.gen_bf16(shape, tau, sigma, scale_log2=sl)
        b = ft2_synth.gen_bf16_torch(shape, tau, sigma, scale_log2=sl).view(torch.int16).numpy().view(np.uint16)
        assert np.array_equal(a, b)


def test_distribution_shape():
    a = ft2_synth.gen_bf16((200000,), 0, 2).view(np.uint16)
    v = torch.from_numpy(a.view(np.int16)).view(torch.bfloat16).double()
    assert 1.1 < v.std().item() < 1.4 and v.abs().max().item() < 256
    assert 0.25 < v[v.abs() < 2].std().item() < 0.33
    assert np.isfinite(v.numpy()).all()


def test_outlier_free_variant_matches_bulk_and_agrees_across_backends():
    # outliers=False keeps every element's bulk draw and drops only the planted
    # 2^-10 outliers; numpy and torch builds agree bit for bit
    import torch
    a = ft2_synth.gen_bf16((300, 700), tau=5, sigma=9)
    b = ft2_synth.gen_bf16((300, 700), tau=5, sigma=9, outliers=False)
    t = ft2_synth.gen_bf16_torch((300, 700), 5, 9, outliers=False).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(b, t)
    va = a.astype(np.uint32) << 16
    vb = b.astype(np.uint32) << 16
    fa, fb = va.view(np.float32), vb.view(np.float32)
    same = fa == fb
    assert 0.0005 < 1 - same.mean() < 0.002          # ~2^-10 of the elements differ
    assert np.all(np.abs(fb) < 1.0)                  # bulk: |z| * 2^-17 < 1
    d = ~same
    ratio = np.abs(fa[d] / fb[d])
    assert np.all(np.isin(np.round(np.log2(ratio)).astype(int), [5, 6, 7, 8]))
