"""Numerics of co-running tenants, in the launch configuration bench.py times
(per layer, on the layer's own GPU input; PAPER.md L276:
the squad barrier).

Per config C2/C3/C4 and per policy (BLESS with per-tenant launcher threads,
BLESS with the single launch thread, STATIC), several "waves": new random
inputs, every activation buffer poisoned with NaN, one request per tenant
submitted (simultaneously, then staggered), drained, and EVERY layer of every
tenant compared with the float64 oracle at the north-star tolerance (bf16:
max relative error 1e-2, reading R24).  A kernel that reads its input before
its producer wrote it (PDL ordering, light exits), a split-K workspace that is
not re-zeroed between launches, or co-resident tenants corrupting each other
all surface as NaN or wrong values.

BLESS runs also check the squad barrier from the launch log: a kernel of squad
s+1 never claims its first tile before every other tenant's last kernel of
squad s has finished (its stream waits on their events).  A kernel may start
during its own stream predecessor's tail: programmatic dependent launch
overlaps the prologue, and data reads wait in griddepcontrol.wait."""
import os

import numpy as np
import pytest
import torch

from oracle.sched_ref import Active, Params, Prof, decide_ref
from synth import profile as sp
from tests.layer_check import check_layer

pytestmark = pytest.mark.gpu

from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi, models  # noqa: E402


@pytest.fixture(scope="module", params=["C2", "C3", "C4"])
def world(request, tmp_path_factory):
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    cfg = request.param
    ctx = capi.Ctx(0)
    ms = models.build_config(ctx, cfg, "bf16")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=1)
    path = str(tmp_path_factory.mktemp(cfg) / "profile.txt")
    ctx.save_profile(path)
    yield cfg, ctx, ms, Prof(sp.load(path))
    ctx.close()


def new_inputs(ms, seed):
    g = torch.Generator(device="cuda").manual_seed(seed)
    for m in ms:
        x = m.input
        if x.dtype.is_floating_point:
            x.copy_(torch.randn(x.shape, generator=g, device="cuda", dtype=torch.float32).to(x.dtype))
        else:
            x.copy_(torch.randint(0, 30522, x.shape, generator=g, device="cuda", dtype=x.dtype))


def poison(ms):
    for m in ms:
        for layer in m.layers:
            if layer.y.dtype.is_floating_point:
                layer.y.fill_(float("nan"))


def run_wave(ctx, ms, policy, stagger_ns, squad_max, split_pct=25, barrier=0):
    p = capi.default_params(policy=policy, squad_max=squad_max, split_pct=split_pct, barrier=barrier)
    ctx.reset(p)
    ctx.start()
    base = capi.now_ns() + 2_000_000
    ids = [ctx.submit(m.tenant, base + j * stagger_ns) for j, m in enumerate(ms)]
    ctx.drain(int(120e9))
    ctx.stop()
    for r in ids:
        assert ctx.poll(r)[0] == capi.BL_OK
    torch.cuda.synchronize()
    return ctx.decisions(), ctx.launches()


def check_all_layers(ms, tag):
    worst = 0.0
    for m in ms:
        for k, layer in enumerate(m.layers):
            err, tol = check_layer(layer, "bf16")
            assert np.isfinite(err) and err <= tol, (tag, m.name, k, layer.kind, layer.name, err)
            worst = max(worst, err)
    return worst


def squads_of(decisions, launches):
    """Launch records grouped by decision (the engine logs a squad's launches in pick order)."""
    out, i = [], 0
    for d in decisions:
        out.append(launches[i:i + d.n_picks])
        i += d.n_picks
    assert i == len(launches)
    return out


def check_squad_barrier(decisions, launches, res_ns=64, join_solo=False):
    """join_solo (bl_params.barrier bit 1, reading R38): a squad that follows
    a solo NSP squad may start beside it and is not checked against it."""
    sq = squads_of(decisions, launches)
    n_pairs = 0
    for (da, a), b in zip(zip(decisions, sq), sq[1:]):
        if join_solo and da.n_part == 1 and not da.config_sp:
            continue
        end_by_tenant = {}
        for r in a:
            assert r.end_ns > 0 and r.nsm > 0, (r.tenant, r.kernel)
            end_by_tenant[r.tenant] = max(end_by_tenant.get(r.tenant, 0), r.end_ns)
        for r in b:
            others = [e for t, e in end_by_tenant.items() if t != r.tenant]
            if others:
                assert r.start_ns >= max(others) - res_ns, (
                    "squad barrier broken", r.tenant, r.kernel, r.start_ns - max(others))
                n_pairs += 1
    return n_pairs


def check_range_barrier(decisions, launches, res_ns=64):
    """bl_params.barrier = 1 (reading R37): a launch of tenant j in squad s+1
    never starts before the end of another tenant's latest chain whose kernels
    used a logical SM that j's chain in squad s+1 uses."""
    last, n_pairs = {}, 0
    for ls in squads_of(decisions, launches):
        umask = {}
        for r in ls:
            assert r.end_ns > 0 and r.nsm > 0, (r.tenant, r.kernel)
            umask[r.tenant] = umask.get(r.tenant, 0) | (((1 << (r.hi - r.lo)) - 1) << r.lo)
        for r in ls:
            for t, (e, msk) in last.items():
                if t != r.tenant and msk & umask[r.tenant]:
                    assert r.start_ns >= e - res_ns, ("range barrier broken", r.tenant, r.kernel, r.start_ns - e)
                    n_pairs += 1
        for t, msk in umask.items():
            last[t] = (max(r.end_ns for r in ls if r.tenant == t), msk)
    return n_pairs


@pytest.mark.parametrize("policy", ["BLESS", "BLESS_1thread", "BLESS_range", "BLESS_join", "STATIC"])
def test_concurrent_every_layer_vs_oracle(world, policy):
    cfg, ctx, ms, prof = world
    squad_max = {"C2": 20, "C3": 10, "C4": 10}[cfg]
    # BLESS_range: the SM-range barrier (R37) with strict SP squads (c = 100%),
    # where chains on disjoint partitions stop waiting for each other
    # BLESS_join: arrivals join in-flight solo NSP squads at once (R38)
    split_pct, barrier = {"BLESS_range": (100, 1), "BLESS_join": (25, 2)}.get(policy, (25, 0))
    waves = [(0, 11), (60_000, 12)] if policy in ("BLESS", "BLESS_range", "BLESS_join") else [(0, 21)]
    old = os.environ.get("BLESS_LAUNCH_THREADS")
    if policy == "BLESS_1thread":
        os.environ["BLESS_LAUNCH_THREADS"] = "0"
    try:
        for stagger, seed in waves:
            new_inputs(ms, seed)
            poison(ms)
            decisions, launches = run_wave(ctx, ms, "STATIC" if policy == "STATIC" else "BLESS", stagger, squad_max,
                                           split_pct, barrier)
            worst = check_all_layers(ms, (cfg, policy, stagger))
            msg = f"\n{cfg} {policy} stagger={stagger}: {sum(len(m.layers) for m in ms)} layers, worst {worst:.2e}"
            if policy != "STATIC":
                assert decisions
                pairs = (check_range_barrier(decisions, launches) if barrier & 1 else
                         check_squad_barrier(decisions, launches, join_solo=bool(barrier & 2)))
                sp_sq = sum(1 for d in decisions if d.config_sp)
                for rec in decisions:
                    got = capi.decision_to_tuple(rec)
                    ref = decide_ref(got["now"], [Active(*a) for a in got["active"]], prof,
                                     Params(squad_max=squad_max, split_pct=split_pct))
                    assert got["picks"] == [tuple(p) for p in ref.picks] and got["config"] == ref.config
                msg += f"; {len(decisions)} squads ({sp_sq} SP), barrier held on {pairs} cross-squad launches"
            for r in launches:
                bits = [w * 32 + b for w in range(8) for b in range(32) if r.sm_mask[w] >> b & 1]
                assert bits and all(r.lo <= x < r.hi for x in bits) and r.fallback == 0, (r.tenant, r.kernel)
            print(msg)
    finally:
        if old is None:
            os.environ.pop("BLESS_LAUNCH_THREADS", None)
        else:
            os.environ["BLESS_LAUNCH_THREADS"] = old
