"""Pins for fault sites (R6) and injection (R7) -- CPU only.

Pinned against: Philox4x32-10 known-answer vectors (Random123, Salmon et al.
SC'11); PAPER.md L185 / Fig. 7 closed forms (exponent-MSB flip: (1,2) -> NaN,
(0,1) -> huge value); PAPER.md L84 fault models (popcount / field checks);
statistical uniformity (chi-square, "uniformly distributed").
"""
import ml_dtypes
import numpy as np
import pytest

import oracle


def test_philox_known_answers():
    # Random123 kat_vectors: philox4x32_10
    assert oracle.philox4x32_10([0, 0, 0, 0], [0, 0]) == [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]
    ff = 0xFFFFFFFF
    assert oracle.philox4x32_10([ff] * 4, [ff, ff]) == [0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD]
    pi = [0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344]
    assert oracle.philox4x32_10(pi, [0xA4093822, 0x299F31D0]) == [0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]


def _site(step, layer, col, mask, token=0):
    s = np.zeros(1, oracle.SITE_DTYPE)
    s["step"], s["layer"], s["col"], s["xor_mask"], s["token"] = step, layer, col, mask, token
    return s


def _bf(bits):
    return np.asarray(bits, np.uint16).view(ml_dtypes.bfloat16).astype(np.float64)


def test_fig7_exponent_msb_flip_bf16():
    # values in (1,2) and (-2,-1) become NaN under one exponent-MSB flip
    allb = np.arange(65536, dtype=np.uint32).astype(np.uint16)
    v = _bf(allb)
    vuln = allb[((v > 1) & (v < 2)) | ((v < -1) & (v > -2))]
    for b in vuln:
        y = np.array([[b]], np.uint16)
        oracle.inject(y, _site(3, 0, 0, 1 << 14), cur_layer=0, cur_step=3)
        assert oracle.isnan(int(y[0, 0]))
    # and no other finite value becomes NaN from that flip
    other = allb[~(((v > 1) & (v < 2)) | ((v < -1) & (v > -2))) & np.isfinite(v)]
    flipped = other ^ np.uint16(1 << 14)
    assert not np.any(np.isnan(_bf(flipped)) & ~np.isin(other, [0x3F80, 0xBF80]))
    # Fig 7(a)-type extreme values (bf16 closed forms, SURVEY.md 8(c) R6/R7 pins)
    for x, want in [(0x3F00, 2.0 ** 127), (0x3F80, np.inf), (0x4000, 0.0), (0xBF80, -np.inf)]:
        y = np.array([[x]], np.uint16)
        oracle.inject(y, _site(1, 2, 0, 1 << 14), cur_layer=2, cur_step=1)
        assert _bf(y)[0, 0] == want


def test_fig7_fp16_layout_extreme_value():
    # the paper's own FP16 example: exponent-MSB flip of 0.5 gives 32768 (L185, Fig 7)
    h = np.array([0.5, 1.5], np.float16).view(np.uint16).reshape(1, 2).copy()
    s = np.concatenate([_site(4, 1, 0, 1 << 14), _site(4, 1, 1, 1 << 14)])
    oracle.inject(h, s, cur_layer=1, cur_step=4, base_row=np.array([0, 0], np.int32))
    f = h.view(np.float16).astype(np.float64)
    assert f[0, 0] == 32768.0 and np.isnan(f[0, 1])


def test_inject_is_an_involution_and_respects_step_layer():
    y = np.arange(40, dtype=np.uint16).reshape(4, 10)
    s = oracle.make_sites(42, 0, 4, oracle.FAULT_2BIT, [10] * 3, n_steps=5, prompt_len=1)
    for st in range(6):
        for ly in range(3):
            y0 = y.copy()
            oracle.inject(y, s, ly, st)
            oracle.inject(y, s, ly, st)
            assert np.array_equal(y, y0)
    z = y.copy()
    oracle.inject(z, _site(2, 1, 3, 0x10), cur_layer=1, cur_step=1)   # wrong step: no-op
    assert np.array_equal(z, y)


def test_prefill_site_uses_token_row():
    y = np.zeros((6, 4), np.uint16)
    s = _site(0, 0, 2, 0x1, token=3)
    oracle.inject(y, s, cur_layer=0, cur_step=0, base_row=np.array([1], np.int32))
    assert y[4, 2] == 1 and y.sum() == 1


LLAMA7B_WIDTHS = [4096, 4096, 4096, 4096, 11008, 11008, 4096] * 32


@pytest.mark.parametrize("model", [oracle.FAULT_1BIT, oracle.FAULT_2BIT, oracle.FAULT_EXP])
def test_site_masks_follow_fault_model(model):
    s = oracle.make_sites(7, 0, 5000, model, LLAMA7B_WIDTHS, n_steps=32, prompt_len=16)
    pc = np.array([bin(int(m)).count("1") for m in s["xor_mask"]])
    if model == oracle.FAULT_2BIT:
        assert np.all(pc == 2)
    else:
        assert np.all(pc == 1)
    assert np.all(s["xor_mask"] < (1 << 16))
    if model == oracle.FAULT_EXP:
        assert np.all((s["xor_mask"] & 0x7F80) == s["xor_mask"])   # bf16 exponent bits 7..14
    assert np.all(s["col"] < np.array(LLAMA7B_WIDTHS)[s["layer"]])
    assert np.all(s["step"] <= 32)
    assert np.all((s["step"] != 0) | (s["token"] < 16)) and np.all(s["token"][s["step"] != 0] == 0)
    assert np.array_equal(s["trial"], np.arange(5000))


def test_sites_are_deterministic_and_shardable():
    a = oracle.make_sites(42, 0, 1000, oracle.FAULT_1BIT, LLAMA7B_WIDTHS, 32, 16)
    b = np.concatenate([oracle.make_sites(42, r * 125, 125, oracle.FAULT_1BIT, LLAMA7B_WIDTHS, 32, 16)
                        for r in range(8)])
    assert a.tobytes() == b.tobytes()


def _chi2_ok(counts, expected):
    # chi-square with a loose threshold (mean + 6 sd of the chi2 distribution)
    k = len(counts)
    chi2 = float(((counts - expected) ** 2 / expected).sum())
    return chi2 < (k - 1) + 6 * np.sqrt(2 * (k - 1))


def test_site_uniformity_chi2():
    n = 200000
    s = oracle.make_sites(1234, 0, n, oracle.FAULT_1BIT, LLAMA7B_WIDTHS, 32, 16)
    assert _chi2_ok(np.bincount(s["step"], minlength=33), n / 33)
    assert _chi2_ok(np.bincount(s["layer"], minlength=224), n / 224)
    bits = np.log2(s["xor_mask"]).astype(int)
    assert _chi2_ok(np.bincount(bits, minlength=16), n / 16)
    q = s[s["layer"] % 7 == 0]["col"] // 256        # q_proj cols in 16 buckets
    assert _chi2_ok(np.bincount(q, minlength=16), q.size / 16)
    e = oracle.make_sites(99, 0, 80000, oracle.FAULT_EXP, LLAMA7B_WIDTHS, 32, 16)
    assert _chi2_ok(np.bincount(np.log2(e["xor_mask"]).astype(int) - 7, minlength=8), 80000 / 8)


def test_step_policy_one_fault_per_decode_step():
    s = oracle.make_sites(42, 0, 32, oracle.FAULT_1BIT, [768], n_steps=32, prompt_len=16, step_policy=1)
    assert s["step"].tolist() == list(range(1, 33))
    assert np.all(s["layer"] == 0) and np.all(s["col"] < 768)


def test_sites_golden_seed42():
    import os
    rows = [l.split() for l in open(os.path.join(os.path.dirname(__file__), "golden", "r6_sites_seed42.txt"))
            if l.strip() and not l.startswith("#")]
    sites = [oracle.make_sites(42, 0, 3, m, LLAMA7B_WIDTHS, 32, 16) for m in range(3)]
    for r in rows:
        t = int(r[0])
        for m in range(3):
            s = sites[m][t]
            assert (int(s["step"]), int(s["layer"]), int(s["col"])) == (int(r[1]), int(r[2]), int(r[3]))
            assert int(s["xor_mask"]) == int(r[4 + m], 16)


# ---- neuron-uniform (size-weighted) branch of R6, reading A11's flag
# (layer_uniform = 0): every output neuron of every linear layer is equally
# likely ("uniformly distributed location", read over neurons).

def test_neuron_uniform_equal_widths_matches_layer_uniform_layer():
    # With equal widths w the global neuron index g = floor(u1 * L * w / 2^32)
    # lies in layer floor(g / w) = floor(u1 * L / 2^32): exactly the layer the
    # layer-uniform branch draws from the same u1 (floor(floor(a)/w) = floor(a/w)).
    # An off-by-one in the layer walk or a wrong size weighting breaks this.
    n = 20000
    for w, L in [(768, 12), (4096, 224), (1, 7)]:
        lu = oracle.make_sites(5, 0, n, oracle.FAULT_1BIT, [w] * L, 32, 16, layer_uniform=True)
        nu = oracle.make_sites(5, 0, n, oracle.FAULT_1BIT, [w] * L, 32, 16, layer_uniform=False)
        assert np.array_equal(lu["layer"], nu["layer"])
        assert np.all(nu["col"] < w)
        # every other field comes from the other Philox words: identical
        for f in ("step", "token", "xor_mask", "trial", "nbits"):
            assert np.array_equal(lu[f], nu[f])


def _philox_u1(seed, t):
    # word u1 of the first Philox block of trial t (R6 counter layout); the
    # generator itself is pinned by the Random123 known answers above
    return oracle.philox4x32_10([t & 0xFFFFFFFF, t >> 32, 0, 0x46543200], [seed & 0xFFFFFFFF, seed >> 32])[1]


def test_neuron_uniform_hand_computed_sites_three_layers():
    # widths 3 / 5 / 2: 10 neurons; layer boundaries at global indices 3 and 8.
    widths = [3, 5, 2]
    s = oracle.make_sites(11, 0, 64, oracle.FAULT_1BIT, widths, 4, 2, layer_uniform=False)
    for t in range(64):
        g = (_philox_u1(11, t) * 10) >> 32          # uniform global neuron index in [0, 10)
        want = (0, g) if g < 3 else ((1, g - 3) if g < 8 else (2, g - 8))
        assert (int(s["layer"][t]), int(s["col"][t])) == want, t
    # a single layer: the draw is plain neuron-uniform within it
    one = oracle.make_sites(11, 0, 64, oracle.FAULT_1BIT, [10], 4, 2, layer_uniform=False)
    assert np.all(one["layer"] == 0)
    assert [int(c) for c in one["col"]] == [(_philox_u1(11, t) * 10) >> 32 for t in range(64)]


def test_neuron_uniform_chi2_size_weighted():
    # layer frequencies proportional to width (not 1/L), neurons uniform inside
    n = 200000
    widths = [4096, 11008, 4096, 2048, 11008, 768]
    s = oracle.make_sites(2024, 0, n, oracle.FAULT_1BIT, widths, 32, 16, layer_uniform=False)
    w = np.array(widths, np.float64)
    cnt = np.bincount(s["layer"], minlength=len(widths))
    assert _chi2_ok(cnt, n * w / w.sum())
    assert not _chi2_ok(cnt, np.full(len(widths), n / len(widths)))   # layer-uniform would fail
    assert np.all(s["col"] < np.array(widths)[s["layer"]])
    for l in (1, 5):   # columns uniform inside a layer, 16 buckets
        c = s[s["layer"] == l]["col"] * 16 // widths[l]
        assert _chi2_ok(np.bincount(c, minlength=16), c.size / 16)
    # Llama-2-7B geometry (224 layers): up/gate layers get 11008/4096 the hits of q/k/v/o/down
    t = oracle.make_sites(77, 0, n, oracle.FAULT_1BIT, LLAMA7B_WIDTHS, 32, 16, layer_uniform=False)
    kind = np.bincount(t["layer"] % 7, minlength=7)
    wk = np.array(LLAMA7B_WIDTHS[:7], np.float64)
    assert _chi2_ok(kind, n * wk / wk.sum())
    assert np.all(t["col"] < np.array(LLAMA7B_WIDTHS)[t["layer"]])
