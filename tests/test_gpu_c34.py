"""Configs C3 (ResNet50 0.4, VGG16 0.3, BERT-base s128 0.2, MobileNetV2 0.1) and
C4 (BERT-large s384 0.5, ResNet152 0.25, DenseNet121 0.25) at full size:
every kernel vs the float64 oracle on its own GPU input (bf16 tolerance 1e-2),
and a short BLESS run per config with K up to 4 participants: every tile inside
its kernel's SM range, no fallback, decisions bit-exact with the oracle."""
import pytest
import torch

from oracle.sched_ref import Active, Params, Prof, decide_ref
from synth import profile as sp
from tests.layer_check import check_layer

pytestmark = pytest.mark.gpu

from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi, models  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_every_layer_vs_oracle(cfg):
    ctx = capi.Ctx(0)
    ms = models.build_config(ctx, cfg, "bf16")
    worst = {}
    for m in ms:
        for k, layer in enumerate(m.layers):
            ctx.run_kernel(m.tenant, k, 0, 148)
            err, tol = check_layer(layer, "bf16")
            assert err <= tol, (m.name, k, layer.kind, layer.name, err)
            worst[m.name] = max(worst.get(m.name, 0.0), err)
        print(f"\n{cfg} {m.name}: {len(m.layers)} kernels, worst max-rel-err {worst[m.name]:.2e}")
    ctx.close()


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_bless_run_confined_bit_exact(cfg, tmp_path):
    ctx = capi.Ctx(0)
    ms = models.build_config(ctx, cfg, "bf16")
    for m in ms:
        ctx.profile_tenant(m.tenant, reps=1)
    path = str(tmp_path / f"{cfg}.profile")
    ctx.save_profile(path)
    prof = Prof(sp.load(path))
    ctx.start()
    base = capi.now_ns() + 1_000_000
    ids = [ctx.submit(j, base + i * 300_000 + j * 50_000) for i in range(3) for j in range(len(ms))]
    ctx.drain(int(120e9))
    ctx.stop()
    for r in ids:
        assert ctx.poll(r)[0] == capi.BL_OK
    for r in ctx.launches():
        bits = [w * 32 + b for w in range(8) for b in range(32) if r.sm_mask[w] >> b & 1]
        assert bits and all(r.lo <= x < r.hi for x in bits), (r.tenant, r.kernel, r.lo, r.hi)
        assert r.fallback == 0
    recs = ctx.decisions()
    kmax = 0
    for rec in recs:
        got = capi.decision_to_tuple(rec)
        kmax = max(kmax, len(got["parts"]))
        ref = decide_ref(got["now"], [Active(*a) for a in got["active"]], prof, Params(squad_max=50))
        assert got["picks"] == [tuple(p) for p in ref.picks] and got["config"] == ref.config
        assert got["t_hat"] == ref.t_hat
    print(f"\n{cfg}: {len(recs)} decisions bit-exact, max participants {kmax}")
    ctx.close()
