"""Campaign statistics (R9) -- ORACLE, test infrastructure only.

PAPER.md L282 (50 inputs x 500 FI per input, "approximately +-0.00554% -
+-0.368% error margins ... with a 95% confidence interval [32, 33]") and L313
(average SDC-rate reduction).  Reading A14: report both the mean of per-cell
reductions and the pooled ratio.
"""
from __future__ import annotations

import math


def wald_margin(p: float, n: int, z: float = 1.96) -> float:
    """95% Wald margin z * sqrt(p (1 - p) / n) of a proportion."""
    return z * math.sqrt(p * (1.0 - p) / n)


def reduction(p_off: float, p_on: float) -> float:
    """SDC-rate reduction 1 - p_on / p_off."""
    return 1.0 - p_on / p_off if p_off > 0 else float("nan")


def mean_and_pooled_reduction(cells):
    """cells: iterable of (k_off, n_off, k_on, n_on). Returns (mean, pooled)."""
    cells = list(cells)
    per = [reduction(ko / no, kn / nn) for ko, no, kn, nn in cells if ko > 0]
    mean = sum(per) / len(per) if per else float("nan")
    ko = sum(c[0] for c in cells)
    no = sum(c[1] for c in cells)
    kn = sum(c[2] for c in cells)
    nn = sum(c[3] for c in cells)
    pooled = reduction(ko / no, kn / nn) if ko > 0 else float("nan")
    return mean, pooled
