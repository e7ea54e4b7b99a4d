"""Latency metrics of the paper -- TEST INFRASTRUCTURE ONLY.

* average latency per application (L300, L318);
* latency deviation sum_j max(T_sys^j - T_iso^j, 0) (L320; reading R25);
* quota attainment_j = 100 * mean(ISO_j) / mean(sys_j) (reading R25).
Percentiles use the nearest-rank definition.
"""
from __future__ import annotations

import math
from typing import Dict, Sequence


def mean(xs: Sequence[float]) -> float:
    return float(sum(xs)) / len(xs) if xs else float("nan")


def percentile(xs: Sequence[float], p: float) -> float:
    """Nearest-rank percentile: the smallest x with >= p% of values <= x."""
    if not xs:
        return float("nan")
    ys = sorted(xs)
    rank = max(1, math.ceil(p / 100.0 * len(ys)))
    return float(ys[rank - 1])


def attainment(iso_mean: float, sys_mean: float) -> float:
    return 100.0 * iso_mean / sys_mean


def deviation(sys_means: Dict[int, float], iso_means: Dict[int, float]) -> float:
    return sum(max(sys_means[j] - iso_means[j], 0.0) for j in sys_means)
