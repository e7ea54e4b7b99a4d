"""GPU tests of the §8(f) rows on config C2 (VGG11 1/3 + ResNet50 2/3):

* f2 memory-management kernels (reading R31): per-request H2D
  input / D2H output copies through bl_set_tenant_io.  New host inputs, NaN in
  every device buffer, BLESS on the wall clock: the device input equals the
  host input bit for bit, every layer matches the float64 oracle on its own
  input, the host output equals the device output bit for bit, and every
  decision (made with the measured copy times in both predictors) replays
  bit-exactly through the oracle's decide_ref.
* f3 SLO mode (L364-L366, reading R30): QoS targets replace T in the progress
  order; every wall-clock decision replays bit-exactly with the targets.
* TEMPORAL (L41, L302, reading R22): every launch decision the engine logged
  (T-cap and T-wc) replays through the oracle's slice rule
  des.temporal_decide_ref; kernels run in order, one request per tenant.
"""
import numpy as np
import pytest
import torch

from oracle import des
from oracle.sched_ref import Active, Params, Prof, decide_ref
from synth import profile as sp
from synth import trace as tr
from tests.layer_check import check_layer

pytestmark = pytest.mark.gpu

from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi, models  # noqa: E402


@pytest.fixture(scope="module")
def c2():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    ms = models.build_config(ctx, "C2", "bf16")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=1)
    yield ctx, ms
    ctx.close()


def replay_all(ctx, path, params):
    ctx.save_profile(path)
    prof = Prof(sp.load(path))
    recs = ctx.decisions()
    assert recs
    for i, rec in enumerate(recs):
        got = capi.decision_to_tuple(rec)
        ref = decide_ref(got["now"], [Active(*a) for a in got["active"]], prof, params)
        assert got["picks"] == [tuple(p) for p in ref.picks], i
        assert got["config"] == ref.config and got["t_hat"] == ref.t_hat and got["t_nsp"] == ref.t_nsp, i
    return prof, len(recs)


def test_host_io_copies_bless(c2, tmp_path):
    ctx, ms = c2
    g = torch.Generator().manual_seed(7)
    host = []
    for m in ms:
        hin = torch.empty(m.input.shape, dtype=m.input.dtype).pin_memory()
        hin.copy_(torch.randn(m.input.shape, generator=g).to(m.input.dtype))
        hout = torch.zeros(m.output.shape, dtype=m.output.dtype).pin_memory()
        host.append((hin, hout))
        ctx.set_tenant_io(m.tenant, hin.data_ptr(), m.input.data_ptr(), hin.numel() * hin.element_size(),
                          m.output.data_ptr(), hout.data_ptr(), hout.numel() * hout.element_size())
    try:
        for m in ms:
            m.input.fill_(float("nan"))
            for layer in m.layers:
                layer.y.fill_(float("nan"))
        torch.cuda.synchronize()
        params = capi.default_params(policy="BLESS", squad_max=20, split_pct=25)
        ctx.reset(params)
        ctx.start()
        base = capi.now_ns() + 2_000_000
        ids = [ctx.submit(j, base + j * 30_000) for j in range(len(ms))]
        ctx.drain(int(60e9))
        ctx.stop()
        for r in ids:
            st, info = ctx.poll(r)
            assert st == capi.BL_OK and info.finish_ns > info.arrival_ns
        torch.cuda.synchronize()
        for m, (hin, hout) in zip(ms, host):
            assert torch.equal(m.input.cpu().view(torch.int16), hin.view(torch.int16)), m.name
            for k, layer in enumerate(m.layers):
                err, tol = check_layer(layer, "bf16")
                assert np.isfinite(err) and err <= tol, (m.name, k, layer.name, err)
            assert torch.equal(m.output.cpu().view(torch.int16), hout.view(torch.int16)), m.name
        prof, n = replay_all(ctx, str(tmp_path / "io.profile"), Params(squad_max=20, split_pct=25))
        assert all(prof.io_in[j] > 0 and prof.io_out[j] > 0 for j in range(len(ms)))
        print(f"\nhost io: H2D {[prof.io_in[j] for j in range(len(ms))]} ns, "
              f"D2H {[prof.io_out[j] for j in range(len(ms))]} ns; {n} decisions bit-exact")
    finally:
        for m in ms:
            ctx.set_tenant_io(m.tenant, 0, 0, 0, 0, 0, 0)


def test_slo_mode_wall_replay(c2, tmp_path):
    ctx, ms = c2
    ctx.reset(capi.default_params(policy="BLESS", squad_max=20, split_pct=25))
    T = [ctx.tenant_info(m.tenant)[2] for m in ms]
    targets = [int(1.2 * T[0]), int(2.0 * T[1])]
    for m, q in zip(ms, targets):
        ctx.set_slo(m.tenant, q)
    try:
        trace = tr.poisson([2.0 * T[0], 2.0 * T[1]], 30, seed=4)     # rho = 0.5 per tenant
        ctx.start()
        base = capi.now_ns() + 2_000_000
        ids = [(a.tenant, ctx.submit(a.tenant, base + a.arrival_ns)) for a in trace]
        ctx.drain(int(60e9))
        ctx.stop()
        lat = {0: [], 1: []}
        for j, r in ids:
            st, info = ctx.poll(r)
            assert st == capi.BL_OK
            lat[j].append(info.finish_ns - info.arrival_ns)
        prof, n = replay_all(ctx, str(tmp_path / "slo.profile"), Params(squad_max=20, split_pct=25))
        assert prof.slo == targets
        viol = sum(x > targets[j] for j in lat for x in lat[j]) / sum(len(v) for v in lat.values())
        print(f"\nSLO targets {targets} ns: {n} decisions bit-exact, violation {100 * viol:.1f}%")
    finally:
        for m in ms:
            ctx.set_slo(m.tenant, 0)


@pytest.mark.parametrize("wc", [0, 1])
def test_temporal_decisions_replay(c2, wc, tmp_path):
    ctx, ms = c2
    period = 1_000_000
    ctx.reset(capi.default_params(policy="TEMPORAL", temporal_period_ns=period, temporal_work_conserving=wc))
    path = str(tmp_path / "t.profile")
    ctx.save_profile(path)
    prof = Prof(sp.load(path))
    S = prof.S
    T = [prof.T[j] for j in range(len(ms))]
    trace = tr.poisson([3.0 * T[0], 3.0 * T[1]], 12, seed=5)
    ctx.start()
    base = capi.now_ns() + 2_000_000
    ids = [ctx.submit(a.tenant, base + a.arrival_ns) for a in trace]
    ctx.drain(int(120e9))
    ctx.stop()
    for r in ids:
        assert ctx.poll(r)[0] == capi.BL_OK
    log = ctx.temporal_log()
    assert len(log) == sum(prof.m[a.tenant] for a in trace)
    nxt = {}
    for i, rec in enumerate(log):
        work = [bool(rec.work_mask >> q & 1) for q in range(len(ms))]
        ref = des.temporal_decide_ref(rec.t, rec.gpu_free, rec.last_sid, rec.turn, rec.turn_end, work, rec.dur,
                                      period, prof.quota_ppm, bool(wc))
        assert ref is not None and ref["launch"], (i, rec.t, rec.tenant)
        assert ref["tenant"] == rec.tenant and ref["slice_end"] == rec.slice_end, (i, ref, rec.slice_end)
        if not wc:
            assert ref["sid"] == rec.sid, i
        assert rec.dur == prof.t(rec.tenant, rec.kernel, S)
        assert rec.kernel == nxt.get(rec.tenant, 0), i
        nxt[rec.tenant] = (rec.kernel + 1) % prof.m[rec.tenant]
    print(f"\nTEMPORAL {'T-wc' if wc else 'T-cap'}: {len(log)} launch decisions replayed through the R22 rule")


def test_run_squad_and_predict(c2):
    """bl_run_squad executes a given squad (the f1 study's measurement): NSP on
    all SMs and an SP split; every pick's duration is positive, the makespan
    covers the longest chain; bl_predict gives Eq. 2 / Eq. 1 for the same squad."""
    ctx, ms = c2
    ctx.reset(capi.default_params(policy="BLESS", squad_max=20))
    S = ctx.device_info().sm_count
    picks = [(0, k) for k in range(3)] + [(1, k) for k in range(5)]
    nsp, kn = ctx.run_squad([(t, k, 0, S) for t, k in picks], reps=3)
    assert all(x > 0 for x in kn) and nsp >= max(kn)
    split = [(0, 49), (49, S)]
    sp, kn2 = ctx.run_squad([(t, k, *split[t]) for t, k in picks], reps=3)
    assert all(x > 0 for x in kn2) and sp >= max(sum(kn2[:3]), max(kn2[3:])) * 0.5
    pn, ps = ctx.predict(picks), ctx.predict(picks, [12, 25])
    assert pn > 0 and ps > 0
    print(f"\nsquad NSP {nsp / 1e3:.1f} us (Eq. 2 {pn / 1e3:.1f}), SP 49/99 {sp / 1e3:.1f} us (Eq. 1 {ps / 1e3:.1f})")
