"""Latency metrics of the paper -- TEST INFRASTRUCTURE ONLY.

Definitions, each from the passage it cites:

* average latency per application under one quota assignment (PAPER.md L320,
  "the average latency of requests from different applications");
* latency deviation of a system under one quota assignment,
  sum_j max(T_sys^j - T_iso^j, 0), with T_iso^j the application's ISO latency
  at its quota (L320; reading R25: T = the mean request latency);
* average latency deviation = the mean of the deviations over several quota
  assignments (L320, "the average latency deviation across various quota
  assignments"; the quantity L334 reports as 14.3 / 2.1 / 0.6 ms);
* quota attainment_j = 100 * mean(ISO_j) / mean(sys_j) (reading R25; >= 100
  means the application is at or below its ISO latency, L300);
* percentiles by the nearest-rank definition (the smallest value with at
  least p% of the sample at or below it).

Pinned by tests/test_metrics.py against the textbook nearest-rank examples
and the hand-worked deviation fixture tests/golden/e6_metrics.json.
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
    """L320: sum over applications j of max(T_sys^j - T_iso^j, 0)."""
    return sum(max(sys_means[j] - iso_means[j], 0.0) for j in sys_means)


def average_deviation(deviations: Sequence[float]) -> float:
    """L320/L334: the deviation averaged over quota assignments."""
    return mean(deviations)
