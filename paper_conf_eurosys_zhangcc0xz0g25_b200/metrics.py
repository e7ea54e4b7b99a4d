"""Request-latency metrics reported by bench.py (§6.2).

* per application: mean / p50 / p99 latency (nearest-rank percentiles);
* quota attainment_j = 100 * mean(ISO_j) / mean(sys_j) (R25, L300);
* latency deviation = sum_j max(T_sys^j - T_iso^j, 0) (L320), T = mean latency;
* average latency deviation = mean deviation over quota assignments (L320, L334).

Reporting only (host floating point on finished latencies; nothing here feeds
a scheduling decision).  tests/test_metrics.py checks these functions against
the oracle's definitions (oracle/metrics_ref.py) and its pinned fixtures.
"""
from __future__ import annotations

from typing import Dict, Iterable, Mapping, Sequence

import numpy as np


def nearest_rank(xs: Sequence[float], p: float) -> float:
    """Smallest sample value with at least p% of the sample at or below it."""
    a = np.sort(np.asarray(xs, dtype=np.float64))
    if a.size == 0:
        return float("nan")
    k = int(np.ceil(p / 100.0 * a.size))
    return float(a[max(k, 1) - 1])


def summary_ms(lat_ns: Sequence[int]) -> Dict[str, float]:
    """mean / p50 / p99 (ms) and the sample size of one application's latencies."""
    if len(lat_ns) == 0:
        return {}
    a = np.asarray(lat_ns, dtype=np.float64)
    return {"mean_ms": float(a.mean()) / 1e6, "p50_ms": nearest_rank(a, 50) / 1e6,
            "p99_ms": nearest_rank(a, 99) / 1e6, "n": int(a.size)}


def attainment_pct(iso_mean: float, sys_mean: float) -> float:
    return 100.0 * float(iso_mean) / float(sys_mean)


def latency_deviation(sys_mean: Mapping[int, float], iso_mean: Mapping[int, float]) -> float:
    """L320: sum_j max(T_sys^j - T_iso^j, 0) over the applications of one quota assignment."""
    return float(sum(max(float(sys_mean[j]) - float(iso_mean[j]), 0.0) for j in sys_mean))


def average_deviation(devs: Iterable[float]) -> float:
    d = [float(x) for x in devs]
    return float(np.mean(d)) if d else float("nan")
