"""Replicas-only multi-GPU plumbing (PAPER.md L171:
"replicating its runtime components for each active GPU").

Every GPU is an independent sharing domain: its own bl_ctx, tenants,
profile, scheduler thread and trace.  Nothing in a request spans GPUs, so
there is no data-path collective; torch.distributed is used only to line up
the timed region (barrier) and to take the max of the per-rank step time.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Dict, List, Optional

# config C5: GPU g hosts the mix M[g mod 3] of {C2, C3, C4}; configs not yet
# built fall back to C2 (documented in DESIGN.md).
C5_MIX = ["C2", "C3", "C4"]


@dataclass(frozen=True)
class ReplicaPlan:
    rank: int
    world: int
    device: int
    config: str
    trace_seed_offset: int   # per-rank trace seeds: independent arrivals per GPU


def plan(rank: int, world: int, local_rank: int, config: str, available: List[str]) -> ReplicaPlan:
    """Static tenant->GPU placement.  config "C5" maps GPU g to C5_MIX[g % 3]
    (the first available one); any other config is replicated on every GPU."""
    if config == "C5":
        want = C5_MIX[rank % len(C5_MIX)]
        cfg = want if want in available else available[0]
    else:
        cfg = config
    return ReplicaPlan(rank, world, local_rank, cfg, 1000 * rank)


def max_over_ranks(value: float, dist=None, device: Optional[str] = None) -> float:
    """Max of a per-rank scalar (the step time) over all ranks."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64, device=device or "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(values: Dict[str, float], dist=None, device: Optional[str] = None) -> Dict[str, float]:
    """Element-wise sum of per-rank counters (requests, latency sums)."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return dict(values)
    import torch
    keys = sorted(values)
    t = torch.tensor([float(values[k]) for k in keys], dtype=torch.float64, device=device or "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return {k: float(v) for k, v in zip(keys, t.tolist())}
