"""Config C2 (VGG11 quota 1/3 + ResNet50 quota 2/3, bf16, batch 1, 224x224) at
full size, in the launch configuration bench.py times:

* every one of the 72 kernels vs the float64 oracle on the kernel's own GPU
  input (bf16: max relative error <= 1e-2), full GPU and an SP-sized window;
* whole requests under STATIC (quota windows) and BLESS: every tile runs inside
  its kernel's SM range, no launch needs the single-CTA fallback, decisions
  replay bit-exactly through the oracle.
"""
import numpy as np
import pytest
import torch

from oracle.sched_ref import Active, Params, Prof, decide_ref
from synth import profile as sp
from tests.layer_check import check_layer

pytestmark = pytest.mark.gpu

from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi, models  # noqa: E402


@pytest.fixture(scope="module")
def c2():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    ms = models.build_config(ctx, "C2", "bf16")
    yield ctx, ms
    ctx.close()


@pytest.mark.parametrize("lo,hi", [(0, 148), (49, 148)])
def test_c2_every_layer_vs_oracle(c2, lo, hi):
    ctx, ms = c2
    worst = {}
    for m in ms:
        for k, layer in enumerate(m.layers):
            ctx.run_kernel(m.tenant, k, lo, hi)
            err, tol = check_layer(layer, "bf16")
            assert err <= tol, (m.name, k, layer.name, err)
            worst[m.name] = max(worst.get(m.name, 0.0), err)
    print("\nworst max-rel-err per model:", worst)


def _flat_profile(ctx, ms, S):
    # scheduling inputs only (STATIC ignores them; BLESS needs a complete table)
    for m in ms:
        for k in range(len(m.layers)):
            ctx.set_profile_row(m.tenant, k, [max(2000, 300000 // s) for s in range(1, S + 1)], S)


def _mask_bits(r):
    return [w * 32 + b for w in range(8) for b in range(32) if r.sm_mask[w] >> b & 1]


@pytest.mark.parametrize("policy", ["STATIC", "UNBOUND", "BLESS", "ISO_burst"])
def test_c2_requests_confined_no_fallback(policy, tmp_path):
    """ISO_burst: 8 requests of each tenant submitted at once, so whole
    requests queue back to back on each tenant's stream (programmatic
    dependent launch keeps the next kernel's CTAs waiting while the quota
    window is still busy) -- the placement-starvation case."""
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    ctx = capi.Ctx(0, policy="ISO" if policy == "ISO_burst" else policy)
    S = ctx.device_info().sm_count
    ms = models.build_config(ctx, "C2", "bf16")
    if policy == "BLESS":
        for m in ms:
            ctx.profile_tenant(m.tenant, reps=2)
    else:
        _flat_profile(ctx, ms, S)
    ctx.start()
    base = capi.now_ns() + 1_000_000
    gap = 0 if policy == "ISO_burst" else 400_000
    ids = [ctx.submit(j, base + i * gap) for i in range(8) for j in range(2)]
    ctx.drain(int(60e9))
    ctx.stop()
    lat = []
    for r in ids:
        st, info = ctx.poll(r)
        assert st == capi.BL_OK
        lat.append(info.finish_ns - info.arrival_ns)
    recs = ctx.launches()
    assert len(recs) == 8 * sum(len(m.layers) for m in ms)
    for r in recs:
        bits = _mask_bits(r)
        assert bits and all(r.lo <= b < r.hi for b in bits), (r.tenant, r.kernel, r.lo, r.hi)
        assert r.fallback == 0, (r.tenant, r.kernel, r.lo, r.hi)
    assert max(lat) < 50e6, max(lat)      # no pathological (fallback-driven) latency
    if policy == "BLESS":
        path = str(tmp_path / "c2.profile")
        ctx.save_profile(path)
        prof = Prof(sp.load(path))
        for rec in ctx.decisions():
            got = capi.decision_to_tuple(rec)
            ref = decide_ref(got["now"], [Active(*a) for a in got["active"]], prof, Params(squad_max=50))
            assert got["picks"] == [tuple(p) for p in ref.picks] and got["config"] == ref.config
    ctx.close()
