"""Protection coverages of PAPER.md Table 1 (L164-L177) on the runner's layer
lists -- CPU only: each scheme's covered layers agree with the oracle's
Table 1 transcription (oracle/critical.py), per architecture."""
import pytest

from oracle import critical
from paper_conf_hpdc_sunzmg00y25_b200.runner import CONFIGS

SCHEME = {"ft2": "FT2", "maximals": "MaxiMals", "globalclipper": "GlobalClipper", "none": "Ranger"}


@pytest.mark.parametrize("model", ["opt-1.3b", "llama-2-7b"])
@pytest.mark.parametrize("cov", sorted(SCHEME))
def test_coverage_matches_table1(model, cov):
    cfg = CONFIGS[model]
    got = {("OUT_PROJ" if n == "o_proj" else n.upper()) for n in cfg.coverage_names(cov)}
    present = {("OUT_PROJ" if n == "o_proj" else n.upper()) for n, _, _, _ in cfg.linears()}
    assert got == critical.TABLE1_COVERAGE[SCHEME[cov]] & present


def test_ft2_coverage_is_the_critical_heuristic_and_all_is_every_linear():
    for cfg in CONFIGS.values():
        assert cfg.coverage_names("ft2") == cfg.critical_names()
        assert cfg.coverage_names("all") == [n for n, _, _, _ in cfg.linears()]
    with pytest.raises(ValueError):
        CONFIGS["opt-1.3b"].coverage_names("ranger++")
