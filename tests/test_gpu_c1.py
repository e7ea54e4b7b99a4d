"""GPU tests (B200 via gpurun): probe, per-kernel parity with the oracle,
SM gating invariants, and the engine end to end on config C1 -- decisions
replayed bit-exactly through the oracle's decide_ref.  Everything goes through
the C ABI (libbless.so)."""
import os

import numpy as np
import pytest
import torch

from oracle import des
from oracle import layers_ref as L
from oracle.sched_ref import Active, Params, Prof, decide_ref
from synth import profile as sp
from synth import trace as tr
from tests.layer_check import check_layer, np64

pytestmark = pytest.mark.gpu

from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi, models  # noqa: E402


@pytest.fixture(scope="module")
def lib_built():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    assert torch.cuda.is_available()
    return True


def mask_bits(rec):
    out = []
    for w in range(8):
        for b in range(32):
            if rec.sm_mask[w] >> b & 1:
                out.append(w * 32 + b)
    return out


def test_probe(lib_built):
    ctx = capi.Ctx(0)
    info = ctx.device_info()
    assert info.sm_count == torch.cuda.get_device_properties(0).multi_processor_count
    assert (info.cc_major, info.cc_minor) == (10, 0)
    lids = sorted(v for v in info.smid_to_lid if v != 255)
    assert lids == list(range(info.sm_count))
    print(f"\nS={info.sm_count} max_smid={info.max_smid} tpc_pairs={info.tpc_pairs_found} "
          f"globaltimer_res={info.globaltimer_res_ns}ns clock_offset={info.clock_offset_ns}")
    ctx.close()


@pytest.mark.parametrize("dtype", ["fp32", "bf16"])
def test_c1_layer_parity_and_gating(lib_built, dtype):
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    ms = models.build_config(ctx, "C1", dtype)
    ranges = [(0, S), (0, 1), (37, 86), (S - 3, S)]
    for m in ms:
        for k, layer in enumerate(m.layers):
            for lo, hi in ranges:
                layer.y.zero_()
                ctx.run_kernel(m.tenant, k, lo, hi)
                err, tol = check_layer(layer, dtype)
                assert err <= tol, (m.name, k, lo, hi, err)
    ctx.close()


def test_gating_invariants(lib_built):
    """Every tile processed on an SM inside the kernel's range; no fallback."""
    ctx = capi.Ctx(0, policy="STATIC")
    S = ctx.device_info().sm_count
    ms = models.build_config(ctx, "C1", "fp32")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=3)
    ctx.start()
    t0 = capi.now_ns()
    for i in range(6):
        for m in ms:
            ctx.submit(m.tenant, t0 + i * 1000)
    ctx.drain(int(20e9))
    ctx.stop()
    recs = ctx.launches()
    assert len(recs) == 6 * sum(len(m.layers) for m in ms)
    for r in recs:
        bits = mask_bits(r)
        assert bits and all(r.lo <= b < r.hi for b in bits), (r.tenant, r.kernel, r.lo, r.hi, bits)
        assert r.fallback == 0
        assert r.end_ns >= r.start_ns > 0
    # STATIC ranges = Hamilton apportionment (R18)
    q0, _, _ = ctx.tenant_info(0)
    assert {(r.lo, r.hi) for r in recs if r.tenant == 0} == {(0, q0)}
    assert {(r.lo, r.hi) for r in recs if r.tenant == 1} == {(q0, S)}
    ctx.close()


def _run_trace(ctx, trace, t_base):
    ids = [ctx.submit(a.tenant, t_base + a.arrival_ns) for a in trace]
    return ids


@pytest.mark.parametrize("dtype,ablate", [("fp32", 0), ("bf16", 0), ("fp32", 1), ("fp32", 2)])
def test_c1_bless_wall_replay_bit_exact(lib_built, dtype, ablate, tmp_path):
    """C1 end to end under BLESS on the wall clock: every request completes,
    every decision replays bit-exactly through decide_ref, all restricted
    kernels stay inside their windows, and the whole-model output matches the
    fp64 oracle forward (fp32: 1e-4, bf16: 1e-2 per layer).  ablate 1/2: the
    §6.8 ablation variants (reading R32) replay bit-exactly as well."""
    ctx = capi.Ctx(0, squad_max=4, ablate=ablate)
    ms = models.build_config(ctx, "C1", dtype)
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=5)
    path = str(tmp_path / "c1.profile")
    ctx.save_profile(path)
    prof = Prof(sp.load(path))
    T = [prof.T[j] for j in range(2)]
    trace = tr.poisson([2.0 * T[0], 2.0 * T[1]], 8, seed=1)        # rho = 0.5
    ctx.start()
    base = capi.now_ns() + 2_000_000
    ids = _run_trace(ctx, trace, base)
    ctx.drain(int(30e9))
    ctx.stop()
    for r in ids:
        st, info = ctx.poll(r)
        assert st == capi.BL_OK and info.finish_ns > info.arrival_ns
    recs = ctx.decisions()
    assert recs
    pr = Params(squad_max=4, ablate=ablate)
    for i, rec in enumerate(recs):
        got = capi.decision_to_tuple(rec)
        ref = decide_ref(got["now"], [Active(*a) for a in got["active"]], prof, pr)
        assert got["picks"] == [tuple(p) for p in ref.picks], i
        assert got["config"] == ref.config and got["t_hat"] == ref.t_hat and got["t_nsp"] == ref.t_nsp, i
    S = prof.S
    for r in ctx.launches():
        bits = mask_bits(r)
        assert all(r.lo <= b < r.hi for b in bits) and r.fallback == 0
    # numerics of the last request of each tenant (buffers hold it): every
    # layer on its own GPU input at the north-star tolerance (R24: 1e-4 fp32,
    # 1e-2 bf16), and for fp32 the whole model end to end at 1e-4 (no
    # per-layer rounding to compound).  bf16 has no end-to-end bound: each
    # layer rounds its output to bf16 (2^-9 relative) and SURVEY §8(c) C-4
    # compares bf16 per layer only.
    for m in ms:
        for k, layer in enumerate(m.layers):
            err, tol = check_layer(layer, dtype)
            assert err <= tol, (m.name, k, err)
        if dtype != "fp32":
            continue
        x = np64(m.input)
        for layer in m.layers:
            if layer.kind == "gemm":
                x = L.gemm(x, np64(layer.w), np64(layer.shift), layer.act)
            else:
                x = L.conv2d_nhwc(x, np64(layer.w), None, np64(layer.shift), 1, 1, 1, layer.act)
        err = L.max_rel_err(np64(m.output).reshape(x.shape), x)
        assert err < 1e-4, (m.name, err)
    ctx.close()


def test_c1_virtual_clock_matches_des(lib_built, tmp_path):
    """VIRTUAL clock on the GPU: the whole decision sequence equals the oracle
    DES on the same trace and profile (R17)."""
    ctx = capi.Ctx(0, squad_max=4, clock=capi.BL_CLOCK_VIRTUAL, squad_overhead_ns=3000)
    ms = models.build_config(ctx, "C1", "fp32")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=3)
    path = str(tmp_path / "c1v.profile")
    ctx.save_profile(path)
    prof = Prof(sp.load(path))
    trace = tr.poisson([2.0 * prof.T[0], 2.0 * prof.T[1]], 8, seed=1)
    ids = [ctx.submit(a.tenant, a.arrival_ns) for a in trace]
    ctx.start()
    ctx.drain(int(30e9))
    recs = ctx.decisions()
    ctx.stop()
    ref = des.run_bless(trace, prof, Params(squad_max=4, squad_overhead_ns=3000))
    assert len(recs) == len(ref.decisions)
    for rec, d in zip(recs, ref.decisions):
        got = capi.decision_to_tuple(rec)
        assert got["now"] == d.now and got["picks"] == [tuple(p) for p in d.picks] and got["config"] == d.config
    for r in ids:
        assert ctx.poll(r)[0] == capi.BL_OK
    ctx.close()


@pytest.mark.parametrize("policy", ["STATIC", "UNBOUND", "TEMPORAL"])
def test_baselines_complete(lib_built, policy):
    ctx = capi.Ctx(0, policy=policy, temporal_period_ns=200_000)
    ms = models.build_config(ctx, "C1", "fp32")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=3)
    ctx.start()
    base = capi.now_ns() + 1_000_000
    ids = [ctx.submit(j, base + i * 20_000) for i in range(5) for j in range(2)]
    ctx.drain(int(30e9))
    ctx.stop()
    for r in ids:
        assert ctx.poll(r)[0] == capi.BL_OK
    ctx.close()


def test_linger_steal_path_exact(lib_built, monkeypatch):
    """Executor safety net (executor.cuh gate_linger): an out-of-range CTA that
    sees no in-range claim within linger_ns helps drain the queue (flag bit 1,
    a bounded confinement violation instead of a stall).  With linger 0 the
    path runs on almost every restricted launch: every request still
    completes, every layer matches the oracle, and the steal is reported."""
    monkeypatch.setenv("BLESS_LINGER_NS", "0")
    ctx = capi.Ctx(0, policy="STATIC")
    S = ctx.device_info().sm_count
    ms = models.build_config(ctx, "C1", "fp32")
    for m in ms:
        for k in range(len(m.layers)):
            ctx.set_profile_row(m.tenant, k, [max(2000, 300000 // s) for s in range(1, S + 1)], S)
    ctx.start()
    base = capi.now_ns() + 1_000_000
    ids = [ctx.submit(j, base + i * 50_000) for i in range(4) for j in range(2)]
    ctx.drain(int(20e9))
    ctx.stop()
    for r in ids:
        assert ctx.poll(r)[0] == capi.BL_OK
    recs = ctx.launches()
    steals = sum(1 for r in recs if r.fallback & 2)
    assert steals > 0, "linger 0 should exercise the steal path"
    for m in ms:
        for k, layer in enumerate(m.layers):
            err, tol = check_layer(layer, "fp32")
            assert err <= tol, (m.name, k, err)
    print(f"\nsteal path: {steals}/{len(recs)} launches helped by out-of-range CTAs, outputs exact")
    ctx.close()


def test_stats_ring_wraps_without_stale_records(lib_built, tmp_path, monkeypatch):
    """A run with more launches than the stats-ring window (ADVICE round 1:
    records older than ahead() launches are reused): with a 2^10 ring (ahead =
    512) and ~1,500 launches every request still completes, every launch whose
    record is reported has its SM mask inside its range and no fallback, and
    light launches older than the window are reported as unknown (nsm = -1,
    no times) instead of from a reused record."""
    monkeypatch.setenv("BLESS_STATS_RING_LOG2", "10")
    ctx = capi.Ctx(0, squad_max=4)
    ms = models.build_config(ctx, "C1", "fp32")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=2)
    path = str(tmp_path / "c1.profile")
    ctx.save_profile(path)
    prof = Prof(sp.load(path))
    trace = tr.poisson([2.0 * prof.T[0], 2.0 * prof.T[1]], 320, seed=3)   # 320 requests, 1,600 launches
    ctx.start()
    ids = _run_trace(ctx, trace, capi.now_ns() + 2_000_000)
    ctx.drain(int(60e9))
    ctx.stop()
    for r in ids:
        st, info = ctx.poll(r)
        assert st == capi.BL_OK and info.finish_ns > info.arrival_ns
    recs = ctx.launches()
    assert len(recs) > 1024
    known = [r for r in recs if r.nsm > 0]
    unknown = [r for r in recs if r.nsm < 0]
    assert unknown, "no launch fell out of the 512-launch window"
    assert all(r.start_ns == 0 and r.end_ns == 0 for r in unknown)
    for r in known:
        bits = mask_bits(r)
        assert bits and all(r.lo <= b < r.hi for b in bits) and r.fallback == 0 and r.end_ns >= r.start_ns
    # first and last kernels of every request publish their stamps (full exit
    # protocol) and are harvested during the run, whatever their age
    m_of = [len(m.layers) for m in ms]
    for r in recs:
        if r.kernel == 0 or r.kernel == m_of[r.tenant] - 1:
            assert r.nsm > 0, (r.tenant, r.kernel, r.seq)
    print(f"\n{len(recs)} launches, {len(known)} reported, {len(unknown)} older light launches unknown")
    ctx.close()
