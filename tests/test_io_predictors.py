"""Memory-management kernels in both predictors (PAPER.md
L229, reading R31).  Oracle pin: the hand-worked fixture E5 (in
test_oracle_sched.py) and the closed forms below; product parity: the C++
decide() and the VIRTUAL-clock engine bit-exact with the oracle when the
profile carries per-tenant copy times."""
import dataclasses

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import des
from oracle.sched_ref import Active, Params, Prof, decide_ref, predict_nsp, predict_sp
from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi
from synth import profile as sp
from synth import trace as tr


@pytest.fixture(scope="module", autouse=True)
def built_lib():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)


def with_io(pf, io):
    return sp.ProfileFile(pf.S, pf.g, [dataclasses.replace(tn, io_in=int(a), io_out=int(b))
                                       for tn, (a, b) in zip(pf.tenants, io)])


def _world(seed, K=3, S=16, g=4):
    rng = np.random.Generator(np.random.PCG64(seed))
    tenants = [sp.random_tenant(f"t{j}", 1_000_000 // K, int(rng.integers(1, 8)), S, rng, 2e4, 0.5, 0.3, 200)
               for j in range(K)]
    return sp.ProfileFile(S, g, tenants), rng


@pytest.mark.parametrize("seed", range(10))
def test_io_closed_forms(seed):
    """Whole request in one squad, single participant: Eq. 1 on s SMs =
    sum_k t[k][s] + io_in + io_out; Eq. 2 (one request) = sum_k t[k][min(S, d_k)]
    interpolated + io_in + io_out.  Picks without kernel 0 / the last kernel
    carry no copy time."""
    pf, rng = _world(seed, K=1)
    a, b = int(rng.integers(0, 5000)), int(rng.integers(0, 5000))
    p0, p1 = Prof(pf), Prof(with_io(pf, [(a, b)]))
    m = p0.m[0]
    ks = {0: list(range(m))}
    assert predict_sp(ks, (p0.N,), p1)[0] == predict_sp(ks, (p0.N,), p0)[0] + a + b
    assert predict_nsp(ks, p1)[0] == predict_nsp(ks, p0)[0] + a + b
    if m >= 3:
        mid = {0: list(range(1, m - 1))}
        assert predict_nsp(mid, p1)[0] == predict_nsp(mid, p0)[0]


def _ctx_from(pf, tmp, **kw):
    path = str(tmp / "profile.txt")
    sp.save(path, pf)
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, **kw)
    ctx.load_profile(path)
    return ctx


@settings(max_examples=150, deadline=None)
@given(seed=st.integers(0, 10**6), io=st.lists(st.tuples(st.integers(0, 3000), st.integers(0, 3000)),
                                               min_size=3, max_size=3), smax=st.integers(1, 10))
def test_io_decide_bit_exact(tmp_path_factory, seed, io, smax):
    pf, rng = _world(seed)
    pf = with_io(pf, io)
    prof = Prof(pf)
    ctx = _ctx_from(pf, tmp_path_factory.mktemp("io"), squad_max=smax)
    for _ in range(4):
        act = [(j, int(rng.integers(0, 3000)), int(rng.integers(0, prof.m[j]))) for j in range(3)
               if rng.random() < 0.8 or j == 0]
        now = 3000 + int(rng.integers(0, 30000))
        ref = decide_ref(now, [Active(*x) for x in act], prof, Params(squad_max=smax))
        got = capi.decision_to_tuple(ctx.decide(now, act))
        assert got["picks"] == [tuple(p) for p in ref.picks]
        assert (got["config"], got["t_hat"], got["t_nsp"]) == (ref.config, ref.t_hat, ref.t_nsp)
    ctx.close()


def test_io_profile_roundtrip_and_trace(tmp_path):
    pf, _ = _world(21, K=2, S=148)
    pf = with_io(pf, [(12000, 3000), (40000, 800)])
    ctx = _ctx_from(pf, tmp_path, squad_max=8, squad_overhead_ns=500)
    out = str(tmp_path / "rt.txt")
    ctx.save_profile(out)
    assert open(out).read() == open(str(tmp_path / "profile.txt")).read()
    prof = Prof(pf)
    trace = tr.poisson([prof.T[j] / 0.5 for j in range(2)], 20, seed=4)
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
