"""Deployment admission and multi-GPU placement (§4.2.2;
reading R33), and the f4 SM-count restriction (L420): the oracle's rules
pinned by the hand-worked fixture E7 and invariants, the C++ implementations
(bl_deployment_check, bl_place, bl_params.sm_limit) bit-exact with the oracle."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import deploy_ref as D
from oracle import des
from oracle.sched_ref import Params, Prof
from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi
from synth import profile as sp
from synth import trace as tr
from tests.helpers import load_golden

FX = load_golden("e7_deployment.json")


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)


@pytest.mark.parametrize("case", FX["colocate"])
def test_colocate_fixture(case):
    assert D.colocatable(case["avg_ns"], case["span_x"]) is case["ok"], case["why"]


@pytest.mark.parametrize("case", FX["place"])
def test_place_fixture_oracle_and_native(case):
    args = (case["mem"], case["avg_ns"], case["gpu_free"], case["span_x"])
    assert D.place(*args) == case["expected"], case["derivation"]
    assert capi.place(*args) == case["expected"]


@settings(max_examples=200, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 100), st.integers(1_000, 1_000_000)), min_size=0, max_size=10),
       st.lists(st.integers(0, 300), min_size=1, max_size=5), st.integers(1, 60))
def test_place_native_equals_oracle(apps, gpus, span):
    mem = [a[0] for a in apps]
    avg = [a[1] for a in apps]
    got = capi.place(mem, avg, gpus, span)
    assert got == D.place(mem, avg, gpus, span)
    # invariants: memory never over-committed, every GPU's set satisfies the span rule
    for g in range(len(gpus)):
        mine = [i for i, x in enumerate(got) if x == g]
        assert sum(mem[i] for i in mine) <= gpus[g]
        assert D.colocatable([avg[i] for i in mine], span)


def test_deployment_check_native(tmp_path):
    rng = np.random.Generator(np.random.PCG64(3))
    tenants = [sp.random_tenant("short", 500000, 40, 148, rng, 2e5, 0.5, 0.2, 1500),
               sp.random_tenant("long", 500000, 4, 148, rng, 4e6, 0.5, 0.2, 1500)]
    pf = sp.ProfileFile(148, 4, tenants)
    path = str(tmp_path / "p.txt")
    sp.save(path, pf)
    prof = Prof(pf)
    avg = [prof.T[j] // prof.m[j] for j in range(2)]
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL)
    ctx.load_profile(path)
    for span in (5, 30, 1000):
        for free in (10, 100, 1000):
            want = D.deployment_check(avg, [40, 50], free, span)
            assert ctx.deployment_check([40, 50], free, span) == want
    with pytest.raises(capi.BlessError):          # a device-less ctx cannot query free memory
        ctx.deployment_check([1, 1], 0, 30)
    ctx.close()


def _truncate(pf, S2):
    ten = [sp.TenantRows(t.name, t.quota_ppm, [sp.KernelRow(k.name, min(k.d, S2), list(k.t[:S2]))
                                               for k in t.kernels], t.slo_ns, t.io_in, t.io_out)
           for t in pf.tenants]
    return sp.ProfileFile(S2, pf.g, ten)


@pytest.mark.parametrize("S2", [40, 76, 112])
def test_sm_limit_restricts_whole_system(tmp_path, S2):
    """L420 (SM-count sweep): with sm_limit the scheduler sees a GPU of S2 SMs
    -- decisions and model completions equal the oracle DES on the profile
    truncated to S2 columns, every range inside [0, S2)."""
    rng = np.random.Generator(np.random.PCG64(8))
    tenants = [sp.random_tenant("a", 500000, 20, 148, rng, 4e5, 0.8, 0.1, 1500),
               sp.random_tenant("b", 500000, 30, 148, rng, 3e5, 0.8, 0.1, 1500)]
    pf = sp.ProfileFile(148, 4, tenants)
    path = str(tmp_path / "p.txt")
    sp.save(path, pf)
    ctx = capi.Ctx(capi.BL_DEVICE_NONE, clock=capi.BL_CLOCK_VIRTUAL, squad_overhead_ns=2000, sm_limit=S2)
    ctx.load_profile(path)
    small = Prof(_truncate(pf, S2))
    trace = tr.poisson([small.T[j] / 0.4 for j in range(2)], 10, seed=2)
    ids = [ctx.submit(a.tenant, a.arrival_ns) for a in trace]
    ctx.start()
    ctx.drain(int(30e9))
    recs = ctx.decisions()
    ref = des.run_bless(trace, small, Params(squad_overhead_ns=2000))
    assert len(recs) == len(ref.decisions)
    for r, d in zip(recs, ref.decisions):
        got = capi.decision_to_tuple(r)
        assert got["picks"] == [tuple(p) for p in d.picks] and got["config"] == d.config
        assert all(0 <= lo < hi <= S2 for _, _, lo, hi in got["picks"])
    assert [ctx.poll(r)[1].finish_ns for r in ids] == [ref.finish[i] for i in range(len(trace))]
    ctx.stop()
    assert ctx.tenant_info(0)[0] == Prof(pf).quota_sms[0]     # whole-GPU profile back after the run
    ctx.close()
