"""Request-arrival traces (seeded, integer nanoseconds).

The paper evaluates with closed-loop loads, a Twitter trace and an Azure trace
(Table 2).  The traces are not available offline, so the
build uses synthetic Poisson (C1-C3, C5) and bursty MMPP-2 (C4) arrivals
(SURVEY.md §8(d)).  Arrival times are drawn as float64 with numpy PCG64 and
rounded to int64 ns exactly once, here; nothing downstream re-draws them.

Ordering contract: sorted by arrival, ties by tenant id,
then by file order.
"""
from __future__ import annotations

import json
from dataclasses import dataclass
from typing import Iterable, List, Sequence

import numpy as np


@dataclass(frozen=True)
class Arrival:
    arrival_ns: int
    tenant: int


def _sort(arrs: Iterable[Arrival]) -> List[Arrival]:
    indexed = list(enumerate(arrs))
    indexed.sort(key=lambda p: (p[1].arrival_ns, p[1].tenant, p[0]))
    return [a for _, a in indexed]


def poisson(mean_gap_ns: Sequence[float], n_per_tenant: int | Sequence[int], seed: int,
            start_ns: int = 0) -> List[Arrival]:
    """Independent per-tenant Poisson processes.

    ``mean_gap_ns[j]`` is tenant j's mean inter-arrival gap (1/lambda_j).
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    if isinstance(n_per_tenant, int):
        n_per_tenant = [n_per_tenant] * len(mean_gap_ns)
    out: List[Arrival] = []
    for j, (gap, n) in enumerate(zip(mean_gap_ns, n_per_tenant)):
        gaps = rng.exponential(float(gap), size=int(n))
        times = np.rint(np.cumsum(gaps)).astype(np.int64) + int(start_ns)
        out.extend(Arrival(int(t), j) for t in times)
    return _sort(out)


def simultaneous(n_tenants: int, n_rounds: int, round_gap_ns: int, start_ns: int = 0) -> List[Arrival]:
    """All tenants submit together every ``round_gap_ns`` (the Fig. 4(b) /
    Fig. 15 "arrive at the same time" micro-case)."""
    out = [Arrival(int(start_ns + r * round_gap_ns), j) for r in range(n_rounds) for j in range(n_tenants)]
    return _sort(out)


def mmpp2(mean_gap_ns: Sequence[float], n_per_tenant: int, seed: int, on_frac: float = 0.2,
          on_mult: float = 4.0, off_mult: float = 0.25, on_dwell_ns: float = 20e6,
          off_dwell_ns: float = 80e6) -> List[Arrival]:
    """Bursty two-state Markov-modulated Poisson arrivals per tenant (config C4).

    ON state rate = on_mult * lambda, OFF state rate = off_mult * lambda,
    exponential dwell times with the given means.  ``on_frac`` is recorded for
    documentation only (it equals on_dwell/(on_dwell+off_dwell) by default).
    """
    del on_frac
    rng = np.random.Generator(np.random.PCG64(seed))
    out: List[Arrival] = []
    for j, gap in enumerate(mean_gap_ns):
        lam = 1.0 / float(gap)
        t = 0.0
        on = bool(rng.random() < on_dwell_ns / (on_dwell_ns + off_dwell_ns))
        state_end = rng.exponential(on_dwell_ns if on else off_dwell_ns)
        times = []
        while len(times) < n_per_tenant:
            rate = lam * (on_mult if on else off_mult)
            dt = rng.exponential(1.0 / rate)
            if t + dt > state_end:
                t = state_end
                on = not on
                state_end = t + rng.exponential(on_dwell_ns if on else off_dwell_ns)
                continue
            t += dt
            times.append(t)
        out.extend(Arrival(int(v), j) for v in np.rint(np.asarray(times)).astype(np.int64))
    return _sort(out)


@dataclass(frozen=True)
class BoxArrival:
    """One request of the box-wide trace: GPU, tenant, time."""
    arrival_ns: int
    gpu: int
    tenant: int


def box_trace(per_gpu_gaps: Sequence[Sequence[float]], n_per_tenant: int, seed: int,
              bursty: Sequence[bool] = ()) -> List[BoxArrival]:
    """Box-wide merge of per-GPU traces (config C5).  GPU g's tenants draw
    their own Poisson (or, if bursty[g], MMPP-2) arrivals from seed
    seed * 1000 + g, so GPU g's slice of the box trace does not depend on how
    many GPUs the box has; the merge is sorted by (arrival, gpu, tenant)."""
    out = []
    for g, gaps in enumerate(per_gpu_gaps):
        sub_seed = seed * 1000 + g
        sub = mmpp2(gaps, n_per_tenant, sub_seed) if (g < len(bursty) and bursty[g]) else \
            poisson(gaps, n_per_tenant, sub_seed)
        out.extend(BoxArrival(a.arrival_ns, g, a.tenant) for a in sub)
    out.sort(key=lambda a: (a.arrival_ns, a.gpu, a.tenant))
    return out


def gpu_slice(box: Sequence[BoxArrival], gpu: int) -> List[Arrival]:
    """GPU g's requests of a box trace (the dispatcher's routing)."""
    return [Arrival(a.arrival_ns, a.tenant) for a in box if a.gpu == gpu]


def save(path: str, arrs: Sequence[Arrival]) -> None:
    with open(path, "w") as f:
        for a in arrs:
            f.write(json.dumps({"arrival_ns": int(a.arrival_ns), "tenant": int(a.tenant)}) + "\n")


def load(path: str) -> List[Arrival]:
    out = []
    with open(path) as f:
        for line in f:
            line = line.strip()
            if line:
                d = json.loads(line)
                out.append(Arrival(int(d["arrival_ns"]), int(d["tenant"])))
    return out
