"""Oracle for BLESS's runtime scheduling decision -- TEST INFRASTRUCTURE ONLY.

Plain Python integers throughout (arbitrary precision, so every cross-product
and sum is exact; no float ever enters a decision -- SURVEY.md §7 principle 1).
Exact ratios are compared with ``fractions.Fraction``.  The argmin over SP
configurations is done by *plain lexicographic enumeration* of the
configuration space, which is the definition; the product uses
an exact DP instead and must agree bit for bit.

Citations are PAPER.md line numbers; readings R1..R26 are DESIGN.md §3
(inherited from SURVEY.md §8(c)).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from fractions import Fraction
from typing import Dict, Iterator, List, Optional, Sequence, Tuple

from synth.profile import ProfileFile

PPM = 1_000_000


# ----------------------------------------------------------------------------
# Registration: quota -> SMs ("n% of the GPU"; reading R18)
# ----------------------------------------------------------------------------
def hamilton(quota_ppm: Sequence[int], S: int) -> List[int]:
    """Largest-remainder (Hamilton) apportionment of S SMs by quota.

    Seats H = round-half-up(S * sum(ppm) / 1e6), capped at S.  Every tenant
    first gets floor(S*ppm_j/1e6); the H - sum(floors) leftover seats go to the
    largest remainders S*ppm_j mod 1e6, ties to the smaller tenant id (R18).
    """
    total = sum(quota_ppm)
    H = min(S, (S * total + PPM // 2) // PPM)
    exact = [S * q for q in quota_ppm]           # in units of 1/PPM SM
    seats = [e // PPM for e in exact]
    rema = [e % PPM for e in exact]
    left = H - sum(seats)
    order = sorted(range(len(quota_ppm)), key=lambda j: (-rema[j], j))
    for j in order[:max(0, left)]:
        seats[j] += 1
    return seats


def static_ranges(quota_sms: Sequence[int]) -> List[Tuple[int, int]]:
    """Contiguous ISO/STATIC SM ranges in tenant-id order (R18)."""
    out, lo = [], 0
    for s in quota_sms:
        out.append((lo, lo + s))
        lo += s
    return out


# ----------------------------------------------------------------------------
# The profile (§4.2.1, Table 1)
# ----------------------------------------------------------------------------
class Prof:
    """t[j][k][s] for s = 1..S, d[j][k], quota_sms, tau, T.

    tau[j][k] = "the duration from the beginning of the application to the
    end of k" with n% SMs (L157): measured along an isolated run of the
    request when the profile carries it for the tenant's quota SMs (reading
    R35: a "tau <sms> ..." line with sms == quota_sms), else
    sum_{i<=k} t[j][i][quota_sms_j};  T[j] = tau[j][m_j - 1] ("isolated
    latency T[n%]", L157).
    """

    def __init__(self, pf: ProfileFile):
        self.S, self.g = pf.S, pf.g
        self.N = pf.S // pf.g                      # number of partitions (L159; R8)
        self.names = [tn.name for tn in pf.tenants]
        self.quota_ppm = [tn.quota_ppm for tn in pf.tenants]
        self.quota_sms = hamilton(self.quota_ppm, self.S)
        self.ntenants = len(pf.tenants)
        self.m = [len(tn.kernels) for tn in pf.tenants]
        self.d = [[k.d for k in tn.kernels] for tn in pf.tenants]
        self._t = [[list(k.t) for k in tn.kernels] for tn in pf.tenants]
        self.tau: List[List[int]] = []
        for j, tn in enumerate(pf.tenants):
            measured = list(getattr(tn, "tau", []) or [])
            if measured and len(measured) == self.m[j] and getattr(tn, "tau_sms", 0) == self.quota_sms[j]:
                self.tau.append(measured)          # R35: measured along an isolated run
                continue
            acc, row = 0, []
            for k in range(self.m[j]):
                acc += self.t(j, k, self.quota_sms[j])
                row.append(acc)
            self.tau.append(row)
        self.T = [row[-1] if row else 0 for row in self.tau]
        # SLO mode (§6.5): "replacing the isolated latency
        # T[n%] in §4.3.1 with the required QoS target".  In P~ = P_r / P_e,
        # P_r = t_e / SLO and P_e = tau / T, so P~ = t_e / (tau * SLO / T);
        # reading R30 floors tau * SLO / T to integer ns.  No SLO: tau itself.
        self.slo = [int(getattr(tn, "slo_ns", 0)) for tn in pf.tenants]
        # memory-management kernels: per-request H2D before
        # kernel 0 and D2H after the last kernel, copy-engine ns
        self.io_in = [int(getattr(tn, "io_in", 0)) for tn in pf.tenants]
        self.io_out = [int(getattr(tn, "io_out", 0)) for tn in pf.tenants]
        self.tau_prog: List[List[int]] = []
        for j in range(self.ntenants):
            if self.slo[j] > 0 and self.T[j] > 0:
                self.tau_prog.append([tk * self.slo[j] // self.T[j] for tk in self.tau[j]])
            else:
                self.tau_prog.append(list(self.tau[j]))

    def t(self, j: int, k: int, s: int) -> int:
        assert 1 <= s <= self.S, s
        return self._t[j][k][s - 1]

    def io(self, j: int, k: int) -> int:
        """L229: "the durations of memory management kernels (e.g., H2D, D2H
        memcpy) are added" in both predictors.  Reading R31: the request's
        input copy belongs to its kernel 0, its output copy to its last kernel."""
        return (self.io_in[j] if k == 0 else 0) + (self.io_out[j] if k == self.m[j] - 1 else 0)


@dataclass
class Params:
    squad_max: int = 50        # max kernels per squad (L181, L408; R5)
    split_pct: int = 50        # Semi-SP split ratio c% (L255, L410; R16)
    seed_all: bool = True      # every active request seeded first (R6)
    squad_overhead_ns: int = 0  # DES only: GPU idle per squad switch (L432)
    # Ablation (§6.8; reading R32): bit 0 = no multi-task scheduler
    # (picks taken round-robin over the active requests in tenant-id order,
    # one kernel each per round, no progress ordering); bit 1 = no execution
    # configuration determiner (no search: every squad runs NSP on [0, S)).
    ablate: int = 0
    # Reading R36: a squad with a single active request closes after
    # min(squad_max, squad_max_solo) kernels (L57 / L121: an arriving request
    # should get its share "instantly"; squads are waited for lazily, so a
    # short solo squad bounds the wait).  0 = squad_max.
    squad_max_solo: int = 0

    @staticmethod
    def from_dict(d: dict) -> "Params":
        return Params(int(d.get("squad_max", 50)), int(d.get("split_pct", 50)),
                      bool(d.get("seed_all", True)), int(d.get("squad_overhead_ns", 0)), int(d.get("ablate", 0)),
                      int(d.get("squad_max_solo", 0)))


@dataclass(frozen=True)
class Active:
    tenant: int
    arrival: int
    next_kernel: int


@dataclass
class Decision:
    now: int
    active: List[Active]
    picks: List[Tuple[int, int, int, int]]          # (tenant, kernel, lo, hi) in pick order
    participants: List[int]                          # sorted tenant ids
    config: Optional[Tuple[int, ...]]                # None = NSP, else p (partitions per participant)
    t_hat: int
    t_nsp: int
    chain_end: Dict[int, int] = field(default_factory=dict)   # predicted end of each participant's picks


# ----------------------------------------------------------------------------
# §4.3.1 request progress perception (L177-L179), readings R1-R4, R20
# ----------------------------------------------------------------------------
def behind_key(now: int, tenant: int, arrival: int, tau_done: int):
    """Sort key: smaller key == more behind == more urgent.

    The paper's relative progress is P~ = P_r / P_e with P_r = t_e/T and
    P_e = tau/T (L179); T cancels, so P~ = t_e / tau.  R1: the request that is
    "falling behind" is the one with the largest t_e/tau (least work done per
    unit of elapsed time).  R2/R20: t_e = now - arrival (clamped at 0).  R3:
    tau = 0 (nothing scheduled yet) means infinitely behind.  R4 ties: smaller
    tau, then earlier arrival, then smaller tenant id.
    """
    te = max(0, now - arrival)
    if tau_done == 0:
        ratio_rank = (0, Fraction(0))                 # +inf ratio sorts first
    else:
        ratio_rank = (1, -Fraction(te, tau_done))     # larger ratio sorts first
    return (ratio_rank, tau_done, arrival, tenant)


# ----------------------------------------------------------------------------
# §4.3.2 squad generation (L181-L187, Fig. 6), readings R5-R7
# ----------------------------------------------------------------------------
def generate_squad(now: int, active: Sequence[Active], prof: Prof, params: Params) -> List[Tuple[int, int]]:
    """Return the ordered picks [(tenant, kernel)] of one kernel squad."""
    nxt = {a.tenant: a.next_kernel for a in active}
    arr = {a.tenant: a.arrival for a in active}

    def tau_done(j: int) -> int:
        # pace of the request: tau (default) or tau * SLO / T (SLO mode, R30)
        return 0 if nxt[j] == 0 else prof.tau_prog[j][nxt[j] - 1]

    def key(j: int):
        return behind_key(now, j, arr[j], tau_done(j))

    picks: List[Tuple[int, int]] = []
    cap = params.squad_max
    if len(active) == 1 and params.squad_max_solo > 0:     # R36
        cap = min(params.squad_max, params.squad_max_solo)

    def pick(j: int) -> bool:
        """Append kernel nxt_j of request j; True when the squad must close:
        (1) the count reached the maximum (R5, inclusive cap) or (2) the
        picked kernel is the request's last kernel (L181; R7)."""
        k = nxt[j]
        picks.append((j, k))
        nxt[j] = k + 1
        return len(picks) >= cap or k == prof.m[j] - 1

    closed = False
    tenants = sorted(nxt)
    if params.ablate & 1:
        # §6.8 "BLESS without the multi-task scheduler can not dynamically
        # control the kernel number from each active request" (L426): equal
        # shares, one kernel per active request per round, tenant-id order;
        # the same closing rules (R5, R7).
        while not closed:
            for j in tenants:
                if nxt[j] < prof.m[j] and pick(j):
                    closed = True
                    break
        return picks
    if params.seed_all and len(tenants) >= 2:             # R6
        for j in sorted(tenants, key=key):
            if pick(j):
                closed = True
                break
    while not closed:
        cands = [j for j in tenants if nxt[j] < prof.m[j]]
        j = min(cands, key=key)                           # "shortest relative progress" (L181)
        closed = pick(j)
    return picks


# ----------------------------------------------------------------------------
# §4.4 execution configuration determiner (L191-L237)
# ----------------------------------------------------------------------------
def per_participant(picks: Sequence[Tuple[int, int]]) -> Dict[int, List[int]]:
    ks: Dict[int, List[int]] = {}
    for j, k in picks:
        ks.setdefault(j, []).append(k)
    return ks


def predict_nsp(ks: Dict[int, List[int]], prof: Prof) -> Tuple[int, List[int]]:
    """Workload-equivalence predictor, Eq. 2 (L222-L227), reading R12.

    Level i (i = 0..q-1, q = max picks per request) overlaps the i-th kernel of
    every request that has one (R_i).  The level's kernels run "sequentially
    where every kernel occupies all active SMs" x_i = min(S, sum_j d(k_i^j)).
    A kernel that "cannot utilize so many SMs" (x > d) is interpolated by work
    equivalence: floor(t[k][d] * d / x).  Returns (t_hat, cumulative level ends).
    """
    parts = sorted(ks)
    q = max(len(ks[j]) for j in parts)
    total, ends = 0, []
    for i in range(q):
        R = [j for j in parts if len(ks[j]) > i]
        x = min(prof.S, sum(prof.d[j][ks[j][i]] for j in R))
        level = 0
        for j in R:
            k = ks[j][i]
            dk = prof.d[j][k]
            if x <= dk:
                level += prof.t(j, k, x)
            else:
                level += (prof.t(j, k, dk) * dk) // x
            level += prof.io(j, k)                      # L229, R31
        total += level
        ends.append(total)
    return total, ends


def sp_sms(p: Sequence[int], idx: int, prof: Prof) -> int:
    """SMs of participant idx under composition p: g*p_idx, except the last
    participant, which takes everything left (S - g*sum of the others)."""
    if idx < len(p) - 1:
        return prof.g * p[idx]
    return prof.S - prof.g * sum(p[:-1])


def predict_sp(ks: Dict[int, List[int]], p: Sequence[int], prof: Prof) -> Tuple[int, Dict[int, int]]:
    """Interference-free predictor, Eq. 1 (L209-L212):
    t_hat = max_j sum_i t[n^j%][k_i^j]."""
    parts = sorted(ks)
    chains = {}
    for idx, j in enumerate(parts):
        s = sp_sms(p, idx, prof)
        chains[j] = sum(prof.t(j, k, s) + prof.io(j, k) for k in ks[j])   # L229, R31
    return max(chains.values()), chains


def compositions(N: int, K: int) -> Iterator[Tuple[int, ...]]:
    """All (p_1..p_K), p_i >= 1, sum = N, in lexicographic order.  Their number
    is C(N-1, K-1) (L205; readings R9, R10)."""
    if K == 1:
        yield (N,)
        return
    for first in range(1, N - K + 2):
        for rest in compositions(N - first, K - 1):
            yield (first,) + rest


def choose_config(ks: Dict[int, List[int]], prof: Prof, search: bool = True) -> Tuple[Optional[Tuple[int, ...]], int, int]:
    """argmin over {NSP} U {all strict spatial splits} (L205, L237).

    R13: NSP is the incumbent and is replaced only by a strictly smaller
    prediction.  R14: compositions are visited in lexicographic order and
    replace the incumbent only if strictly smaller, so the lexicographically
    smallest optimal split wins.  K = 1 => NSP.
    Returns (config or None for NSP, t_hat, t_nsp).
    """
    t_nsp, _ = predict_nsp(ks, prof)
    K = len(ks)
    best, best_t = None, t_nsp
    if K >= 2 and search:   # search = False: the §6.8 ablation without the determiner (R32)
        parts = sorted(ks)
        memo: Dict[Tuple[int, int], int] = {}   # (participant, s) -> sum_i t[k_i][s]; same Eq. 1 terms

        def chain(j: int, s: int) -> int:
            if (j, s) not in memo:
                memo[(j, s)] = sum(prof.t(j, k, s) + prof.io(j, k) for k in ks[j])
            return memo[(j, s)]

        for p in compositions(prof.N, K):
            v = max(chain(j, sp_sms(p, idx, prof)) for idx, j in enumerate(parts))
            if v < best_t:
                best, best_t = p, v
    return best, best_t, t_nsp


def semi_sp_ranges(picks: Sequence[Tuple[int, int]], parts: Sequence[int], config, prof: Prof,
                   split_pct: int) -> List[Tuple[int, int, int, int]]:
    """Semi-SP range plan (L203, L253-L255; reading R16).

    SP: participant idx's window is [g*sum_{l<idx} p_l, g*sum_{l<=idx} p_l),
    the last window extended to S.  Its first r = ceil(m_j * c / 100) picked
    kernels run inside the window; the rest run on [0, S).  NSP: all [0, S).
    """
    S = prof.S
    if config is None:
        return [(j, k, 0, S) for j, k in picks]
    win, lo = {}, 0
    for idx, j in enumerate(parts):
        hi = S if idx == len(parts) - 1 else lo + prof.g * config[idx]
        win[j] = (lo, hi)
        lo = hi
    ks = per_participant(picks)
    r = {j: (len(ks[j]) * split_pct + 99) // 100 for j in parts}
    seen = {j: 0 for j in parts}
    out = []
    for j, k in picks:
        lo_j, hi_j = win[j] if seen[j] < r[j] else (0, S)
        seen[j] += 1
        out.append((j, k, lo_j, hi_j))
    return out


def decide_ref(now: int, active: Sequence[Active], prof: Prof, params: Params) -> Decision:
    """One scheduling round: progress -> squad -> configuration -> ranges."""
    act = sorted(active, key=lambda a: a.tenant)
    assert act, "decide_ref needs at least one active request"
    assert len({a.tenant for a in act}) == len(act), "one active request per tenant (L145)"
    for a in act:
        assert 0 <= a.next_kernel < prof.m[a.tenant]
    picks = generate_squad(now, act, prof, params)
    ks = per_participant(picks)
    parts = sorted(ks)
    config, t_hat, t_nsp = choose_config(ks, prof, search=not (params.ablate & 2))
    ranged = semi_sp_ranges(picks, parts, config, prof, params.split_pct)
    if config is None:
        _, ends = predict_nsp(ks, prof)
        chain = {j: ends[len(ks[j]) - 1] for j in parts}
    else:
        _, chain = predict_sp(ks, config, prof)
    return Decision(now, list(act), ranged, parts, config, t_hat, t_nsp, chain)
