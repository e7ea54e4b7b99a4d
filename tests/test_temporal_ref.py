"""TEMPORAL baseline rule (reading R22; "allocates GPU time
slices ... based on each application's quota", L302 "round-robin time slice
scheduling"): the oracle's stateless per-decision rule temporal_decide_ref is
pinned by hand-worked cases and must reproduce every launch decision the
oracle's own event-driven model (des.run_temporal) makes -- two independent
formulations of the same rule.  The GPU engine's logged decisions are replayed
through the same rule in tests/test_gpu_io_slo_temporal.py."""
import random

import pytest

from oracle import des
from oracle.sched_ref import Prof
from synth import profile as sp
from synth import trace as tr

P = 1000
Q = [250_000, 750_000]      # slices 250 / 750 ns, offsets 0 / 250


def test_slices_hand_worked():
    assert des.temporal_slices(P, Q) == ([250, 750], [0, 250])
    assert des.temporal_slices(2_000_000, [333_333, 666_667]) == ([666_666, 1_333_334], [0, 666_666])


def test_tcap_hand_worked():
    # t = 1100: cycle 1, position 100 -> tenant 0's slice [1000, 1250), id 1*2 + 0
    r = des.temporal_decide_ref(1100, 1000, -1, -1, 0, [True, True], 100, P, Q, False)
    assert r == {"tenant": 0, "slice_end": 1250, "sid": 2, "new_turn": False, "first": True, "launch": True}
    # same slice, not its first launch: 1100 + 200 > 1250 does not fit
    r = des.temporal_decide_ref(1100, 1000, 2, -1, 0, [True, True], 200, P, Q, False)
    assert r["launch"] is False and r["first"] is False
    # ... but the slice's first kernel always starts (non-preemptive overrun)
    r = des.temporal_decide_ref(1100, 1000, 1, -1, 0, [True, True], 200, P, Q, False)
    assert r["launch"] is True
    # GPU busy past the slice end: nothing starts
    r = des.temporal_decide_ref(1100, 1260, 1, -1, 0, [True, True], 10, P, Q, False)
    assert r["launch"] is False
    # t = 1300 -> tenant 1's slice [1250, 2000), id 3
    r = des.temporal_decide_ref(1300, 1300, 2, -1, 0, [True, True], 100, P, Q, False)
    assert (r["tenant"], r["slice_end"], r["sid"]) == (1, 2000, 3)
    # the owner has no work: its slice stays idle (T-cap is not work conserving)
    assert des.temporal_decide_ref(1100, 1000, -1, -1, 0, [False, True], 100, P, Q, False) is None


def test_twc_hand_worked():
    # no turn yet -> tenant 0 (first with work), turn of 250 from max(t, gpu_free)
    r = des.temporal_decide_ref(100, 120, -1, -1, 0, [True, True], 50, P, Q, True)
    assert (r["tenant"], r["slice_end"], r["new_turn"], r["launch"]) == (0, 370, True, True)
    # the running turn continues while t < its end and its tenant has work
    r = des.temporal_decide_ref(200, 220, 1, 0, 370, [True, True], 100, P, Q, True)
    assert (r["tenant"], r["slice_end"], r["new_turn"], r["launch"]) == (0, 370, False, True)
    r = des.temporal_decide_ref(300, 320, 1, 0, 370, [True, True], 100, P, Q, True)
    assert r["launch"] is False          # 320 + 100 > 370, not the turn's first kernel
    # turn over -> the next tenant after 0 with work
    r = des.temporal_decide_ref(400, 400, 1, 0, 370, [True, True], 100, P, Q, True)
    assert (r["tenant"], r["slice_end"], r["new_turn"]) == (1, 1150, True)
    # idle tenants are skipped: turn 1 ends early when it has no work
    r = des.temporal_decide_ref(500, 500, 2, 1, 1150, [True, False], 100, P, Q, True)
    assert (r["tenant"], r["slice_end"]) == (0, 750)
    assert des.temporal_decide_ref(500, 500, 2, 1, 1150, [False, False], 100, P, Q, True) is None


def _prof(seed):
    rng = random.Random(seed)
    S = 16
    tenants = []
    for j in range(rng.randint(2, 4)):
        rows = [sp.KernelRow(f"k{k}", S, [rng.randint(20, 400)] * S) for k in range(rng.randint(1, 6))]
        tenants.append(sp.TenantRows(f"t{j}", 0, rows))
    ppm = [rng.randint(3, 10) for _ in tenants]   # >= 1 SM each at S = 16
    tot = sum(ppm)
    for t, p in zip(tenants, ppm):
        t.quota_ppm = p * 1_000_000 // tot
    return Prof(sp.ProfileFile(S, 1, tenants))


@pytest.mark.parametrize("wc", [False, True])
@pytest.mark.parametrize("seed", range(8))
def test_des_decisions_replay_through_rule(wc, seed):
    prof = _prof(seed)
    period = random.Random(seed).choice([600, 1500, 4000])
    gaps = [prof.T[j] * random.Random(seed + j).uniform(1.0, 4.0) for j in range(prof.ntenants)]
    trace = tr.poisson(gaps, 25, seed=seed + 1)
    log = []
    res = des.run_temporal(trace, prof, period, wc, log=log)
    assert len(res.finish) == len(trace)
    assert log
    nxt = {}
    for rec in log:
        ref = des.temporal_decide_ref(rec["t"], rec["gpu_free"], rec["last_sid"], rec["turn"], rec["turn_end"],
                                      rec["work"], rec["dur"], period, prof.quota_ppm, wc)
        assert ref is not None and ref["launch"], rec
        assert ref["tenant"] == rec["tenant"] and ref["slice_end"] == rec["slice_end"], (ref, rec)
        if not wc:
            assert ref["sid"] == rec["sid"]
        j = rec["tenant"]
        assert rec["kernel"] == nxt.get(j, 0)          # kernels in order, requests one at a time
        nxt[j] = (rec["kernel"] + 1) % prof.m[j]
