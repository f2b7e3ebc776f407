"""Pins for critical-layer selection (R1) and campaign statistics (R9) -- CPU.

R1 is pinned to Table 1: the heuristic of L212 must
reproduce the "Critical Layer" column on both architectures of Fig. 1.
R9 is pinned to the paper's CI margin (+-0.368% at worst, with
n = 50 x 500 = 25 000 and the worst-case SDC rate 9.79% of L317).
"""
import pytest

from oracle import critical, stats


@pytest.mark.parametrize("arch", ["opt", "gptj", "llama", "qwen2"])
def test_table1_reproduced(arch):
    got = critical.critical_layers(arch)
    for node, crit in got.items():
        assert crit == critical.TABLE1_CRITICAL[critical.TABLE1_NAME[node]], (arch, node)


def test_table1_every_row_covered():
    seen = set()
    for arch in ("opt", "llama"):
        seen |= {critical.TABLE1_NAME[n] for n in critical.critical_layers(arch)}
    assert seen == set(critical.TABLE1_CRITICAL)


def test_ft2_covers_exactly_critical_layers():
    crit = {k for k, v in critical.TABLE1_CRITICAL.items() if v}
    assert critical.TABLE1_COVERAGE["FT2"] == crit
    for other in ("Ranger", "MaxiMals", "GlobalClipper"):
        assert critical.TABLE1_COVERAGE[other] < crit   # strict subsets (L164)


def test_protected_layer_counts_match_memory_overhead():
    # 288-512 B = 2 bounds x 2 B x 72..128 protected layers
    per_block = {a: sum(critical.critical_layers(a).values()) for a in ("opt", "llama")}
    assert per_block == {"opt": 3, "llama": 4}
    assert 32 * per_block["llama"] * 2 * 2 == 512          # Llama2-7B / Vicuna-7B
    assert 24 * per_block["opt"] * 2 * 2 == 288            # OPT-1.3B-sized (reading A15)


def test_wald_margin_reproduces_paper():
    assert round(100 * stats.wald_margin(0.0979, 25000), 3) == 0.368
    lo = stats.wald_margin(0.00002, 25000) * 100
    assert 0.004 < lo < 0.007                              # L282 lower margin 0.00554%


def test_reduction_mean_and_pooled():
    m, p = stats.mean_and_pooled_reduction([(10, 100, 1, 100), (20, 100, 10, 100)])
    assert abs(m - 0.7) < 1e-12 and abs(p - (1 - 11 / 30)) < 1e-12
