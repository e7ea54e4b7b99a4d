"""SLO mode (§6.5): the QoS target replaces
the isolated latency T[n%] of §4.3.1, i.e. the progress order paces a tenant
against tau' = floor(tau * slo / T) (reading R30).

Oracle pins (CPU): the hand-worked fixture E4, and the special cases that
reduce to the default policy (slo = T, slo = c*T for every tenant).  Product
parity (CPU, C ABI on a CUDA-free context): single decisions and whole
VIRTUAL-clock traces bit-exact with the oracle for random SLOs.
"""
import dataclasses

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import des
from oracle.sched_ref import Active, Params, Prof, decide_ref, generate_squad
from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi
from synth import profile as sp
from synth import trace as tr
from tests.helpers import golden_profile, load_golden


@pytest.fixture(scope="module", autouse=True)
def built_lib():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)


def with_slo(pf, slos):
    return sp.ProfileFile(pf.S, pf.g, [dataclasses.replace(tn, slo_ns=int(q)) for tn, q in zip(pf.tenants, slos)])


def test_slo_golden_e4():
    fx = load_golden("e4_slo_progress.json")
    base = golden_profile(fx)
    for case in fx["cases"]:
        prof = Prof(with_slo(base, case["slo"]))
        act = [Active(0, 0, 1), Active(1, 0, 1)]
        got = generate_squad(1000, act, prof, Params(squad_max=fx["squad_max"], seed_all=False))
        assert [list(p) for p in got] == case["picks"], case


def _random_world(seed, K=3, S=16, g=4):
    rng = np.random.Generator(np.random.PCG64(seed))
    tenants = [sp.random_tenant(f"t{j}", 1_000_000 // K, int(rng.integers(2, 9)), S, rng, 2e4, 0.5, 0.3, 200)
               for j in range(K)]
    return sp.ProfileFile(S, g, tenants), rng


@pytest.mark.parametrize("seed", range(20))
def test_slo_equal_to_T_or_scaled_is_default_policy(seed):
    """slo_j = T_j gives tau' = tau exactly; slo_j = c*T_j for every tenant
    (c integer) scales every tau by c, so every ratio scales by 1/c and every
    tie stays a tie: the decision equals the default policy's."""
    pf, rng = _random_world(seed)
    prof = Prof(pf)
    c = int(rng.integers(2, 6))
    for slos in ([prof.T[j] for j in range(3)], [c * prof.T[j] for j in range(3)]):
        prof_s = Prof(with_slo(pf, slos))
        for _ in range(5):
            act = [Active(j, int(rng.integers(0, 5000)), int(rng.integers(0, prof.m[j]))) for j in range(3)]
            now = 5000 + int(rng.integers(0, 20000))
            a = decide_ref(now, act, prof, Params(squad_max=6))
            b = decide_ref(now, act, prof_s, Params(squad_max=6))
            assert (a.picks, a.config, a.t_hat) == (b.picks, b.config, b.t_hat)


def test_tight_slo_is_scheduled_first():
    """A tenant whose target is tighter than the others' (same progress, same
    arrival) becomes the most-behind request and seeds the squad."""
    pf, rng = _random_world(7)
    prof = Prof(pf)
    for j in range(3):
        slos = [0, 0, 0]
        slos[j] = max(1, prof.T[j] // 4)
        ps = Prof(with_slo(pf, slos))
        act = [Active(i, 0, 1) for i in range(3)]
        now = 10 * max(prof.T)
        first = generate_squad(now, act, ps, Params(squad_max=1, seed_all=False))[0][0]
        # unless another tenant's tau is already 4x smaller than j's scaled tau
        taus = [ps.tau_prog[i][0] for i in range(3)]
        assert first == min(range(3), key=lambda i: (taus[i], i))


def _ctx_from(pf, tmp, **kw):
    path = str(tmp / "profile.txt")
    sp.save(path, pf)
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, **kw)
    ctx.load_profile(path)
    return ctx


@settings(max_examples=150, deadline=None)
@given(seed=st.integers(0, 10**6), f=st.lists(st.integers(0, 400), min_size=3, max_size=3),
       smax=st.integers(1, 10))
def test_slo_decide_bit_exact(tmp_path_factory, seed, f, smax):
    pf, rng = _random_world(seed)
    prof0 = Prof(pf)
    slos = [prof0.T[j] * x // 100 for j, x in enumerate(f)]   # 0..4 T, 0 = no SLO
    pf = with_slo(pf, slos)
    ctx = _ctx_from(pf, tmp_path_factory.mktemp("s"), squad_max=smax)
    prof = Prof(pf)
    for _ in range(4):
        act = [(j, int(rng.integers(0, 3000)), int(rng.integers(0, prof.m[j]))) for j in range(3)
               if rng.random() < 0.8 or j == 0]
        now = 3000 + int(rng.integers(0, 30000))
        ref = decide_ref(now, [Active(*a) for a in act], prof, Params(squad_max=smax))
        got = capi.decision_to_tuple(ctx.decide(now, act))
        assert got["picks"] == [tuple(p) for p in ref.picks]
        assert got["config"] == ref.config and got["t_hat"] == ref.t_hat
    ctx.close()


def test_slo_set_via_capi_and_profile_roundtrip(tmp_path):
    pf, _ = _random_world(3)
    ctx = _ctx_from(pf, tmp_path)
    ctx.set_slo(1, 12345)
    out = str(tmp_path / "rt.txt")
    ctx.save_profile(out)
    assert sp.load(out).tenants[1].slo_ns == 12345 and sp.load(out).tenants[0].slo_ns == 0
    with pytest.raises(capi.BlessError) as e:
        ctx.set_slo(9, 1)
    assert e.value.status == capi.BL_E_INVALID
    with pytest.raises(capi.BlessError) as e:
        ctx.set_slo(0, -1)
    assert e.value.status == capi.BL_E_INVALID
    ctx.close()


def test_slo_whole_trace_virtual_bit_exact(tmp_path):
    """Whole VIRTUAL-clock trace with a tight and a loose target (the §6.5
    experiment's 1.2x / 2x shape): every decision and completion equals the
    oracle DES."""
    pf, _ = _random_world(11, K=2, S=148)
    prof0 = Prof(pf)
    pf = with_slo(pf, [prof0.T[0] * 12 // 10, prof0.T[1] * 2])
    prof = Prof(pf)
    trace = tr.poisson([prof.T[j] / 0.6 for j in range(2)], 25, seed=2)
    params = dict(squad_max=8, split_pct=50, seed_all=1, squad_overhead_ns=500)
    ctx = _ctx_from(pf, tmp_path, **params)
    ids = [ctx.submit(a.tenant, a.arrival_ns) for a in trace]
    ctx.start()
    ctx.drain(int(30e9))
    fin = [ctx.poll(r)[1] for r in ids]
    recs = ctx.decisions()
    ctx.stop()
    ref = des.run_bless(trace, prof, Params(8, 50, True, 500))
    assert len(recs) == len(ref.decisions)
    for r, d in zip(recs, ref.decisions):
        got = capi.decision_to_tuple(r)
        assert got["picks"] == [tuple(p) for p in d.picks] and got["config"] == d.config
    for i, inf in enumerate(fin):
        assert (inf.start_ns, inf.finish_ns) == (ref.start[i], ref.finish[i])
    ctx.close()
