"""Discrete-event CPU model of the BLESS runtime -- TEST INFRASTRUCTURE ONLY.

Drives ``decide_ref`` on a virtual clock over a request trace (SURVEY.md §8(c)
C-3, reading R17 "VIRTUAL" mode):

* at each decision: admit arrivals <= now into per-tenant FIFO queues; the
  head of each queue becomes the tenant's single active request (L145);
* if nothing is active, jump to the next arrival;
* decide a squad; advance now += t_hat + squad_overhead_ns;
* a request completes at now_before + (the predicted end of its own picks in
  the squad): SP -> its Eq. 1 chain; NSP -> the end of its last Eq. 2 level.

Also ISO/STATIC (Lindley recursion with service T_j, L300) and the TEMPORAL
time-slice models T-cap / T-wc (L41, L302; reading R22).  The model latencies
are context; what must be bit-exact on the product side are the decisions.
"""
from __future__ import annotations

from collections import deque
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence

from synth.trace import Arrival

from .sched_ref import Active, Decision, Params, Prof, decide_ref


@dataclass
class DesResult:
    decisions: List[Decision]
    # per request index (trace order): (tenant, arrival, start, finish)
    finish: Dict[int, int] = field(default_factory=dict)
    start: Dict[int, int] = field(default_factory=dict)
    tenant: Dict[int, int] = field(default_factory=dict)
    arrival: Dict[int, int] = field(default_factory=dict)

    def latencies(self, j: Optional[int] = None) -> List[int]:
        return [self.finish[r] - self.arrival[r] for r in sorted(self.finish)
                if j is None or self.tenant[r] == j]


def run_bless(trace: Sequence[Arrival], prof: Prof, params: Params) -> DesResult:
    res = DesResult([])
    queues = {j: deque() for j in range(prof.ntenants)}
    active: Dict[int, List[int]] = {}        # tenant -> [req, arrival, next_kernel]
    now, i, n = 0, 0, len(trace)
    while True:
        while i < n and trace[i].arrival_ns <= now:
            a = trace[i]
            queues[a.tenant].append((i, a.arrival_ns))
            res.tenant[i], res.arrival[i] = a.tenant, a.arrival_ns
            i += 1
        for j in range(prof.ntenants):
            if j not in active and queues[j]:
                r, arr = queues[j].popleft()
                active[j] = [r, arr, 0]
        if not active:
            if i >= n:
                break
            now = trace[i].arrival_ns
            continue
        act = [Active(j, v[1], v[2]) for j, v in sorted(active.items())]
        d = decide_ref(now, act, prof, params)
        res.decisions.append(d)
        counts: Dict[int, int] = {}
        for j, _k, _lo, _hi in d.picks:
            counts[j] = counts.get(j, 0) + 1
        for j, c in counts.items():
            r = active[j][0]
            if active[j][2] == 0:
                res.start[r] = now
            active[j][2] += c
            if active[j][2] == prof.m[j]:
                res.finish[r] = now + d.chain_end[j]
                del active[j]
        now += d.t_hat + params.squad_overhead_ns
    return res


def run_iso(trace: Sequence[Arrival], prof: Prof) -> DesResult:
    """ISO / STATIC model: each tenant alone on its quota SMs, FIFO, service
    T_j (L157, L300).  Lindley: finish_n = max(arrival_n, finish_{n-1}) + T_j."""
    res = DesResult([])
    last = {j: 0 for j in range(prof.ntenants)}
    for r, a in enumerate(trace):
        j = a.tenant
        st = max(a.arrival_ns, last[j])
        res.tenant[r], res.arrival[r], res.start[r] = j, a.arrival_ns, st
        res.finish[r] = st + prof.T[j]
        last[j] = res.finish[r]
    return res


def temporal_slices(period_ns: int, quota_ppm: Sequence[int]):
    """Reading R22 (L41 "allocates GPU time slices to applications ... based on
    each application's quota"): tenant j's slice is period * quota_ppm_j / 1e6
    ns, slices laid out back to back in tenant-id order."""
    lens = [period_ns * q // 1_000_000 for q in quota_ppm]
    offs = [sum(lens[:j]) for j in range(len(lens))]
    return lens, offs


def temporal_decide_ref(t: int, gpu_free: int, last_sid: int, turn: int, turn_end: int, work: Sequence[bool],
                        dur: int, period_ns: int, quota_ppm: Sequence[int], work_conserving: bool):
    """One TEMPORAL launch decision at time t (R22; L41, L302), stated without
    a loop so a wall-clock run's logged decisions can be replayed.

    T-cap: the slice owning t is the one whose [off_j, off_j + len_j) holds
    t mod P; its end is cycle*P + off_j + len_j and its id cycle*n + j.
    T-wc (round robin skipping idle tenants, L302): the running turn continues
    while t < its end and its tenant has work; otherwise the next tenant after
    it in id order that has work starts a turn of len_j when the GPU is free,
    max(t, gpu_free).  A kernel that does not fit ends its turn at once (the
    caller logs the expired turn end), as run_temporal does.
    Admission (non-preemptive kernels): with st = max(gpu_free, t), a kernel
    of duration dur is launched iff st < slice end and (it is the slice's
    first launch or st + dur <= slice end).

    Returns None if no tenant owns t (T-cap idle gap, or no work), else a dict
    {tenant, slice_end, sid (T-cap only; None for T-wc), new_turn, launch}.
    'first' for T-wc is decided by the caller's sid bookkeeping: a new turn is
    always a first launch; a continuing turn is first iff nothing launched in
    it yet (last_sid tells)."""
    n = len(quota_ppm)
    lens, offs = temporal_slices(period_ns, quota_ppm)
    if not work_conserving:
        cyc, pos = t // period_ns, t % period_ns
        owner = [j for j in range(n) if offs[j] <= pos < offs[j] + lens[j]]
        if not owner or not work[owner[0]]:
            return None
        j = owner[0]
        slice_end = cyc * period_ns + offs[j] + lens[j]
        sid = cyc * n + j
        first = sid != last_sid
        new_turn = False
    else:
        if turn < 0 or t >= turn_end or not work[turn]:
            start = -1 if turn < 0 else turn
            pick = next(((start + s) % n for s in range(1, n + 1) if work[(start + s) % n]), None)
            if pick is None:
                return None
            # a turn starts when the GPU is free (run_temporal: t = max(t, end))
            j, slice_end, new_turn = pick, max(t, gpu_free) + lens[pick], True
        else:
            j, slice_end, new_turn = turn, turn_end, False
        sid = None
        first = new_turn
    st = max(gpu_free, t)
    launch = st < slice_end and (first or st + dur <= slice_end)
    return {"tenant": j, "slice_end": slice_end, "sid": sid, "new_turn": new_turn, "first": first,
            "launch": launch}


def run_temporal(trace: Sequence[Arrival], prof: Prof, period_ns: int, work_conserving: bool,
                 log: Optional[list] = None) -> DesResult:
    """TEMPORAL time slicing on the full GPU (L41, L302; reading R22).

    Tenant j's slice length is period * quota_ppm_j / 1e6.  Kernels run one at
    a time on all S SMs with duration t[j][k][S] and are non-preemptive: within
    a slice a kernel is launched only if its predicted end fits in the slice,
    except the slice's first kernel.
    T-cap (work_conserving=False): fixed cyclic slices; an idle tenant's slice
    stays idle.  T-wc (True): round robin that skips tenants with no work; a
    turn ends when its time is up, when its tenant has no work, or when its
    next kernel does not fit (the next tenant with work takes the GPU at once).
    """
    S = prof.S
    nt = prof.ntenants
    res = DesResult([])
    pending = {j: deque() for j in range(nt)}
    for r, a in enumerate(trace):
        pending[a.tenant].append((r, a.arrival_ns))
        res.tenant[r], res.arrival[r] = a.tenant, a.arrival_ns
    slice_len = [period_ns * q // 1_000_000 for q in prof.quota_ppm]
    offs = [sum(slice_len[:j]) for j in range(nt)]
    cur_req: Dict[int, List[int]] = {}       # tenant -> [req, next_kernel]
    remaining = len(trace)
    gpu_free = 0

    def next_arrival(j: int) -> Optional[int]:
        return pending[j][0][1] if pending[j] else None

    state = {"last_sid": -1, "turn": -1, "turn_end": 0, "nofit": False}

    def tenant_has_work(q: int, t: int) -> bool:
        return q in cur_req or (next_arrival(q) is not None and next_arrival(q) <= t)

    def run_slice(j: int, start: int, end: int, sid: int = -1) -> int:
        """Run tenant j from max(start, gpu_free) until its slice ends.
        Returns the time the GPU becomes free (== start if nothing ran).
        With ``log``: one record per launched kernel, in the shape of the
        engine's bl_temporal_rec (replayed by temporal_decide_ref)."""
        nonlocal remaining
        t = start
        first = True
        state["nofit"] = False
        while t < end:
            if j not in cur_req:
                na = next_arrival(j)
                if na is None or na >= end:
                    break
                if na > t:
                    if work_conserving:
                        break        # T-wc skips an idle tenant: its turn ends (R22)
                    t = na
                    continue
                r, _ = pending[j].popleft()
                cur_req[j] = [r, 0]
            r, k = cur_req[j]
            dur = prof.t(j, k, S)
            if not first and t + dur > end:
                state["nofit"] = True
                break
            if log is not None:
                log.append({"t": t, "gpu_free": t, "slice_end": end, "dur": dur, "sid": sid,
                            "last_sid": state["last_sid"], "turn": state["turn"], "turn_end": state["turn_end"],
                            "work": [tenant_has_work(q, t) for q in range(nt)], "tenant": j, "kernel": k})
            state["last_sid"] = sid
            if work_conserving:
                state["turn"], state["turn_end"] = j, end
            if k == 0:
                res.start[r] = t
            t += dur
            first = False
            cur_req[j][1] += 1
            if cur_req[j][1] == prof.m[j]:
                res.finish[r] = t
                del cur_req[j]
                remaining -= 1
        return t

    if not work_conserving:
        cycle = 0
        while remaining > 0:
            base = cycle * period_ns
            # skip empty cycles quickly
            has_work = any(cur_req.get(j) for j in range(nt))
            if not has_work:
                nxt = [next_arrival(j) for j in range(nt) if next_arrival(j) is not None]
                if nxt and min(nxt) >= base + period_ns and min(nxt) > gpu_free:
                    cycle = max(cycle + 1, min(nxt) // period_ns)
                    continue
            for j in range(nt):
                s0 = base + offs[j]
                s1 = s0 + slice_len[j]
                st = max(s0, gpu_free)
                if st >= s1:
                    continue
                gpu_free = max(gpu_free, run_slice(j, st, s1, cycle * nt + j))
            cycle += 1
    else:
        t = 0
        j = 0
        sid_wc = 0
        while remaining > 0:
            has = [j2 for j2 in range(nt)
                   if j2 in cur_req or (next_arrival(j2) is not None and next_arrival(j2) <= t)]
            if not has:
                state["turn"], state["turn_end"] = -1, 0     # nobody has work: no running turn
                t = min(next_arrival(j2) for j2 in range(nt) if next_arrival(j2) is not None)
                continue
            # next tenant in round-robin order starting at j that has work
            for step in range(nt):
                jj = (j + step) % nt
                if jj in has:
                    break
            sid_wc += 1
            end = run_slice(jj, t, t + slice_len[jj], sid_wc)
            if state["turn"] == jj and state["nofit"]:
                state["turn_end"] = end      # a kernel that did not fit ended the turn
            t = max(t, end)
            j = (jj + 1) % nt
    return res
