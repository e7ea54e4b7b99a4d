"""Deployment rules of the paper (§4.2.2) -- TEST INFRASTRUCTURE ONLY.

Reading R33:
* L163: "BLESS avoids placing applications with short kernels and applications
  with extremely long kernels together ... BLESS works well to co-locate most
  deep learning applications, with the average kernel duration varying from
  10us to 300us" -> a set of applications may share a GPU iff the largest
  average kernel duration is at most span_x (= 300/10 = 30) times the smallest;
  an application's average kernel duration is its isolated latency at its
  quota over its kernel count, T_j / m_j (L157 profile quantities);
* L169: "checks the remained memory capacity on the GPU and guarantees that
  the placement would not cause out-of-memory" -> the sum of the
  applications' memory must fit the GPU's free memory;
* L171: "a central controller can leverage the memory requirement and profiled
  kernel information to decide which specific GPU to place applications" ->
  applications in order of decreasing memory (ties: smaller index), each to the
  GPU with the most remaining free memory among those where it fits and keeps
  the duration rule (ties: smaller GPU index); -1 if no GPU can take it.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple


def colocatable(avg_kernel_ns: Sequence[int], span_x: int = 30) -> bool:
    if not avg_kernel_ns:
        return True
    return max(avg_kernel_ns) <= span_x * min(avg_kernel_ns)


def deployment_check(avg_kernel_ns: Sequence[int], mem_bytes: Sequence[int], free_bytes: int,
                     span_x: int = 30) -> Tuple[bool, int]:
    """(admissible, reason): 0 ok, 1 kernel-duration span (L163), 2 memory (L169)."""
    if not colocatable(avg_kernel_ns, span_x):
        return False, 1
    if sum(mem_bytes) > free_bytes:
        return False, 2
    return True, 0


def place(mem_bytes: Sequence[int], avg_kernel_ns: Sequence[int], gpu_free: Sequence[int],
          span_x: int = 30) -> List[int]:
    order = sorted(range(len(mem_bytes)), key=lambda a: (-mem_bytes[a], a))
    left = list(gpu_free)
    on: List[List[int]] = [[] for _ in gpu_free]
    out = [-1] * len(mem_bytes)
    for a in order:
        ok = [g for g in range(len(gpu_free))
              if mem_bytes[a] <= left[g] and colocatable(on[g] + [avg_kernel_ns[a]], span_x)]
        if not ok:
            continue
        best = min(ok, key=lambda g: (-left[g], g))
        out[a] = best
        left[best] -= mem_bytes[a]
        on[best].append(avg_kernel_ns[a])
    return out
