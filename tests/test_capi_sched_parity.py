"""C-ABI library (CPU-only use) and bit-exact parity of the C++ scheduler with
the oracle (SURVEY.md §8(c) "scheduling decisions and SM assignments must be
bit-exact").  Runs on a CUDA-free context (BL_DEVICE_NONE): the same C++
decide() and virtual-clock engine the GPU path uses, no kernels.
"""
import os
import re

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import des
from oracle.sched_ref import Active, Params, Prof, decide_ref
from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi
from synth import profile as sp
from synth import trace as tr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bless", "bless.h")


@pytest.fixture(scope="session", autouse=True)
def built_lib():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)


def test_library_exports_every_declared_symbol():
    src = open(HEADER).read()
    declared = set(re.findall(r"\b(bl_[a-z_]+)\s*\(", src))
    declared -= {"bl_status"}
    L = capi.lib()
    for name in sorted(declared):
        assert hasattr(L, name), name
    assert declared == set(capi.exported_symbols())
    assert b"sm_100a" in L.bl_version()


def test_enum_mirror_matches_header():
    """Every enumerator of bless.h has the same value in the Python binding."""
    src = open(HEADER).read()
    for name, val in re.findall(r"\b(BL_[A-Z0-9_]+)\s*=\s*(-?\d+)", src):
        assert getattr(capi, name) == int(val), name


def _ctx_from(pf, tmp_path, **kw):
    path = str(tmp_path / "profile.txt")
    sp.save(path, pf)
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, **kw)
    ctx.load_profile(path)
    return ctx


def _ref_tuple(d):
    return {"picks": [tuple(p) for p in d.picks], "parts": list(d.participants), "config": d.config,
            "t_hat": d.t_hat, "t_nsp": d.t_nsp}


def _cpp_tuple(rec):
    t = capi.decision_to_tuple(rec)
    return {k: t[k] for k in ("picks", "parts", "config", "t_hat", "t_nsp")}


def test_errors(tmp_path):
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL)
    with pytest.raises(capi.BlessError) as e:
        ctx.register_tenant(1.5, "x")
    assert e.value.status == capi.BL_E_QUOTA
    ctx.register_tenant(0.7, "a")
    with pytest.raises(capi.BlessError) as e:
        ctx.register_tenant(0.4, "b")
    assert e.value.status == capi.BL_E_QUOTA
    with pytest.raises(capi.BlessError) as e:     # no profile yet
        ctx.start()
    assert e.value.status == capi.BL_E_STATE
    with pytest.raises(capi.BlessError) as e:
        ctx.submit(0, 0)
    assert e.value.status == capi.BL_E_STATE
    with pytest.raises(capi.BlessError) as e:
        ctx.poll(12345)
    assert e.value.status == capi.BL_E_NOTFOUND
    with pytest.raises(capi.BlessError) as e:
        ctx.device_info()
    assert e.value.status == capi.BL_E_STATE
    op = capi.bl_op()
    op.kind = capi.BL_OP_GEMM
    with pytest.raises(capi.BlessError) as e:     # device-less ctx takes virtual ops only
        ctx.append_kernel(0, op)
    assert e.value.status == capi.BL_E_INVALID
    ctx.close()


def test_hamilton_and_tau_match_oracle(tmp_path):
    rng = np.random.Generator(np.random.PCG64(9))
    tenants = [sp.random_tenant(f"t{j}", q, 5 + j, 148, rng, 3e5, 0.5, 0.2, 1500)
               for j, q in enumerate([400000, 300000, 200000, 100000])]
    pf = sp.ProfileFile(148, 4, tenants)
    ctx = _ctx_from(pf, tmp_path)
    prof = Prof(pf)
    for j in range(4):
        q, m, T = ctx.tenant_info(j)
        assert (q, m, T) == (prof.quota_sms[j], prof.m[j], prof.T[j])
    # round trip of the profile file through the C++ writer
    out = str(tmp_path / "rt.txt")
    ctx.save_profile(out)
    assert open(out).read() == open(str(tmp_path / "profile.txt")).read()


@st.composite
def world(draw):
    S = draw(st.sampled_from([4, 8, 12, 16, 20]))
    g = draw(st.sampled_from([g for g in (1, 2, 3, 4) if S // g >= 2]))
    K = draw(st.integers(1, 4))
    m = [draw(st.integers(1, 6)) for _ in range(K)]
    seed = draw(st.integers(0, 100000))
    pf = sp.random_table(S, g, [1_000_000 // K] * K, m, seed, tmax=400, noisy=draw(st.booleans()))
    K_act = draw(st.integers(1, K))
    who = sorted(draw(st.permutations(list(range(K))))[:K_act])
    active = [(j, draw(st.integers(0, 300)), draw(st.integers(0, m[j] - 1))) for j in who]
    now = draw(st.integers(0, 1500))
    params = dict(squad_max=draw(st.integers(1, 12)), split_pct=draw(st.sampled_from([0, 30, 50, 75, 100])),
                  seed_all=int(draw(st.booleans())), ablate=draw(st.sampled_from([0, 0, 1, 2, 3])),
                  squad_max_solo=draw(st.sampled_from([0, 0, 1, 2, 5])))
    return pf, active, now, params


@settings(max_examples=250, deadline=None)
@given(world())
def test_decide_bit_exact_small(tmp_path_factory, w):
    pf, active, now, params = w
    tmp = tmp_path_factory.mktemp("d")
    ctx = _ctx_from(pf, tmp, **params)
    ref = decide_ref(now, [Active(*a) for a in active], Prof(pf),
                     Params(params["squad_max"], params["split_pct"], bool(params["seed_all"]),
                            ablate=params["ablate"], squad_max_solo=params["squad_max_solo"]))
    assert _cpp_tuple(ctx.decide(now, active)) == _ref_tuple(ref)
    ctx.close()


@pytest.mark.parametrize("seed", range(6))
def test_decide_bit_exact_b200_scale(tmp_path, seed):
    """S = 148, g = 4 (N = 37, reading R8), K up to 4, squad_max 50: the exact
    DP against the oracle's enumeration of all C(36, K-1) splits."""
    rng = np.random.Generator(np.random.PCG64(100 + seed))
    K = 2 + seed % 3
    quotas = [[333333, 666667], [400000, 300000, 300000], [400000, 300000, 200000, 100000]][K - 2]
    frac = [0.3, 0.6, 0.9][seed % 3]
    tenants = [sp.random_tenant(f"t{j}", quotas[j], int(rng.integers(8, 40)), 148, rng, 4e5, frac, 0.15, 1500)
               for j in range(K)]
    pf = sp.ProfileFile(148, 4, tenants)
    ctx = _ctx_from(pf, tmp_path, squad_max=50)
    prof = Prof(pf)
    for it in range(8):
        active = [(j, int(rng.integers(0, 100000)), int(rng.integers(0, prof.m[j]))) for j in range(K)
                  if rng.random() < 0.85 or j == 0]
        now = 100000 + int(rng.integers(0, 400000))
        ref = decide_ref(now, [Active(*a) for a in active], prof, Params(squad_max=50))
        assert _cpp_tuple(ctx.decide(now, active)) == _ref_tuple(ref), (seed, it)
    ctx.close()


def _virtual_run(ctx, trace):
    ids = [ctx.submit(a.tenant, a.arrival_ns) for a in trace]
    ctx.start()
    ctx.drain(int(30e9))
    out = {}
    for i, r in enumerate(ids):
        stt, info = ctx.poll(r)
        assert stt == capi.BL_OK
        out[i] = (info.start_ns, info.finish_ns)
    recs = ctx.decisions()
    ctx.stop()
    return recs, out


@pytest.mark.parametrize("case", ["fig1_like", "c3_like", "random_small", "ablate_sched", "ablate_both"])
def test_whole_trace_virtual_bit_exact(tmp_path, case):
    """Whole trace, VIRTUAL clock (R17): every decision record (now, admitted
    set, picks, config, SM ranges, predictions) and every model completion time
    equal the oracle DES."""
    rng = np.random.Generator(np.random.PCG64(5))
    if case == "fig1_like":
        S, g = 148, 4
        tenants = [sp.random_tenant("vgg", 333333, 16, S, rng, 5e5, 0.85, 0.1, 1500),
                   sp.random_tenant("r50", 666667, 55, S, rng, 3e5, 0.85, 0.1, 1500)]
        params = dict(squad_max=50, split_pct=50, seed_all=1, squad_overhead_ns=2000)
        n = 30
    elif case == "c3_like":
        S, g = 148, 4
        tenants = [sp.random_tenant(f"t{j}", q, m, S, rng, 3e5, 0.4, 0.15, 1500)
                   for j, (q, m) in enumerate(zip([400000, 300000, 200000, 100000], [55, 21, 30, 25]))]
        params = dict(squad_max=50, split_pct=50, seed_all=1, squad_overhead_ns=2000)
        n = 10
    elif case.startswith("ablate"):   # §6.8 ablation (R32) on a C2-like pair
        S, g = 148, 4
        tenants = [sp.random_tenant("vgg", 333333, 16, S, rng, 5e5, 0.85, 0.1, 1500),
                   sp.random_tenant("r50", 666667, 55, S, rng, 3e5, 0.85, 0.1, 1500)]
        params = dict(squad_max=20, split_pct=25, seed_all=1, squad_overhead_ns=2000,
                      ablate=1 if case == "ablate_sched" else 3)
        n = 20
    else:
        S, g = 16, 4
        tenants = [sp.random_tenant(f"t{j}", q, m, S, rng, 2e4, 0.5, 0.3, 200)
                   for j, (q, m) in enumerate(zip([500000, 250000, 250000], [4, 7, 3]))]
        params = dict(squad_max=5, split_pct=50, seed_all=0, squad_overhead_ns=0)
        n = 40
    pf = sp.ProfileFile(S, g, tenants)
    prof = Prof(pf)
    trace = tr.poisson([prof.T[j] / 0.5 for j in range(len(tenants))], n, seed=1)
    ctx = _ctx_from(pf, tmp_path, **params)
    recs, fin = _virtual_run(ctx, trace)
    ref = des.run_bless(trace, prof, Params(params["squad_max"], params["split_pct"], bool(params["seed_all"]),
                                            params["squad_overhead_ns"], params.get("ablate", 0)))
    assert len(recs) == len(ref.decisions)
    for i, (r, d) in enumerate(zip(recs, ref.decisions)):
        got = capi.decision_to_tuple(r)
        assert got["now"] == d.now, i
        assert got["active"] == [(a.tenant, a.arrival, a.next_kernel) for a in d.active], i
        assert _cpp_tuple(r) == _ref_tuple(d), i
    for i in range(len(trace)):
        assert fin[i] == (ref.start[i], ref.finish[i]), i
    ctx.close()


def test_ablate_out_of_range_rejected():
    """bl_params.ablate outside 0..3 is BL_E_INVALID at bl_create (header)."""
    with pytest.raises(capi.BlessError) as e:
        capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, ablate=4)
    assert e.value.status == capi.BL_E_INVALID


def test_barrier_out_of_range_rejected():
    """bl_params.barrier outside 0..3 is BL_E_INVALID at bl_create and at
    bl_reset (header); 0..3 are accepted."""
    for b in (-1, 4):
        with pytest.raises(capi.BlessError) as e:
            capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, barrier=b)
        assert e.value.status == capi.BL_E_INVALID
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, barrier=1)
    with pytest.raises(capi.BlessError) as e:
        ctx.reset(capi.default_params(clock=capi.BL_CLOCK_VIRTUAL, barrier=5))
    assert e.value.status == capi.BL_E_INVALID
    ctx.reset(capi.default_params(clock=capi.BL_CLOCK_VIRTUAL, barrier=3))
    ctx.reset(capi.default_params(clock=capi.BL_CLOCK_VIRTUAL, barrier=0))
    ctx.close()


@settings(max_examples=150, deadline=None)
@given(world(), st.integers(0, 10_000))
def test_predict_matches_oracle_eq1_eq2(tmp_path_factory, w, pseed):
    """bl_predict (the f1 study's predictor entry point) == the oracle's Eq. 2
    (NSP) and Eq. 1 (any split) on the decision's own squad; the decision's
    t_nsp / t_hat are the same numbers."""
    from oracle.sched_ref import compositions, per_participant, predict_nsp, predict_sp
    pf, active, now, params = w
    path = str(tmp_path_factory.mktemp("pr") / "p.txt")
    sp.save(path, pf)
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, **{**params, "ablate": 0})
    ctx.load_profile(path)
    prof = Prof(pf)
    rec = ctx.decide(now, active)
    got = capi.decision_to_tuple(rec)
    picks = [(t, k) for t, k, _, _ in got["picks"]]
    ks = per_participant(picks)
    assert ctx.predict(picks) == predict_nsp(ks, prof)[0] == got["t_nsp"]
    K = len(ks)
    if K >= 2:
        comps = list(compositions(prof.N, K))
        rng = np.random.Generator(np.random.PCG64(pseed))
        for i in rng.choice(len(comps), size=min(8, len(comps)), replace=False):
            p = comps[int(i)]
            assert ctx.predict(picks, list(p)) == predict_sp(ks, p, prof)[0]
        if got["config"] is not None:
            assert ctx.predict(picks, list(got["config"])) == got["t_hat"]
    with pytest.raises(capi.BlessError):
        ctx.predict(picks, [prof.N + 1] + [1] * (K - 1))
    ns, npk = ctx.time_decide([rec], reps=2)
    assert ns > 0 and npk == 2 * len(picks)
    ctx.close()


@settings(max_examples=120, deadline=None)
@given(world(), st.integers(0, 10_000), st.booleans())
def test_measured_tau_bit_exact(tmp_path_factory, w, seed, match):
    """Reading R35 (tau[n%][k] is "the duration from the
    beginning of the application to the end of k", T[n%] its isolated
    latency): a profile carrying a measured "tau" line per tenant.  With
    tau_sms == quota SMs both sides use it for the progress order and T;
    with another SM count both fall back to the prefix sums.  Decisions stay
    bit-exact, the C++ writer round-trips the line."""
    from synth.profile import load, save
    pf, active, now, params = w
    prof0 = Prof(pf)
    rng = np.random.Generator(np.random.PCG64(seed))
    for j, tn in enumerate(pf.tenants):
        steps = rng.integers(1, 500, size=len(tn.kernels))
        tn.tau = [int(v) for v in np.cumsum(steps)]
        tn.tau_sms = prof0.quota_sms[j] if match else prof0.quota_sms[j] + 1
    d = tmp_path_factory.mktemp("tau")
    path = str(d / "p.txt")
    save(path, pf)
    prof = Prof(load(path))
    for j, tn in enumerate(pf.tenants):
        want = tn.tau if match else prof0.tau[j]
        assert prof.tau[j] == want and prof.T[j] == want[-1]
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, **params)
    ctx.load_profile(path)
    for j in range(len(pf.tenants)):
        assert ctx.tenant_info(j)[2] == prof.T[j]
    got = _cpp_tuple(ctx.decide(now, active))
    ref = decide_ref(now, [Active(*a) for a in active], prof, Params(**params))
    assert got == _ref_tuple(ref)
    out = str(d / "rt.txt")
    ctx.save_profile(out)
    assert open(out).read() == open(path).read()
    ctx.close()
