"""Replicas-only multi-GPU plumbing (PAPER.md L171:
"replicating its runtime components for each active GPU").

Every GPU is an independent sharing domain: its own bl_ctx, tenants, profile
and scheduler.  Nothing in a request spans GPUs, so there is no data-path
collective and no NCCL.  A box-wide trace (synth.trace.box_trace) is routed to
the GPUs by a static tenant->GPU placement:

* one process for the whole box: one bl_ctx per GPU and one native dispatcher
  thread (bl_dispatch) that hands each request to its GPU's ctx at its arrival
  time;
* one process per GPU (torchrun, as the driver launches bench.py): every rank
  builds the same box trace and dispatches its own GPU's slice; the ranks meet
  only on the host (gloo, CPU tensors) for the barrier around the timed region,
  the max of the step time and the whole-job sums.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Dict, List, Optional, Sequence

# config C5: GPU g hosts the mix M[g mod 3] of {C2, C3, C4}
C5_MIX = ["C2", "C3", "C4"]


@dataclass(frozen=True)
class ReplicaPlan:
    gpu: int          # index of the GPU in the box (torchrun rank, or device index in one process)
    config: str


def plan(gpu: int, config: str) -> ReplicaPlan:
    """Static tenant->GPU placement: "C5" maps GPU g to C5_MIX[g % 3]; any
    other config is replicated on every GPU."""
    return ReplicaPlan(gpu, C5_MIX[gpu % len(C5_MIX)] if config == "C5" else config)


def dispatch_entries(box, gpu_to_ctx: Dict[int, int]):
    """(ctx index, tenant, arrival) for the box requests of the GPUs this
    process owns, in arrival order (input of capi.dispatch)."""
    return [(gpu_to_ctx[a.gpu], a.tenant, a.arrival_ns) for a in box if a.gpu in gpu_to_ctx]


def barrier(dist=None):
    if dist is not None and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()


def max_over_ranks(value: float, dist=None) -> float:
    """Max of a per-rank scalar (the step time) over all ranks (host-side gloo)."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(values: Dict[str, float], dist=None) -> Dict[str, float]:
    """Element-wise sum of per-rank counters (requests, latency sums)."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return dict(values)
    import torch
    keys = sorted(values)
    t = torch.tensor([float(values[k]) for k in keys], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return {k: float(v) for k, v in zip(keys, t.tolist())}


def gather(obj, dist=None) -> List:
    """All ranks' objects (e.g. per-GPU T_iso lists for the box trace)."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return [obj]
    out: List = [None] * dist.get_world_size()
    dist.all_gather_object(out, obj)
    return out
