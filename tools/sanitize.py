"""Small-shape workload for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck) over the executor and the tenant kernels: one bf16
tenant with a tcgen05 GEMM, per-tap and halo tcgen05 convs, split-K, the fused
tcgen05 attention, pooling, LayerNorm and the SIMT kernels, each launched on
the whole GPU and on a restricted SM window, then a short BLESS run of C1
(engine, light exits, squad barriers).

  compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    build.build(verbose=False)
    os.environ["BLESS_TC_AUTOTUNE"] = "0"
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    t = ctx.register_tenant(1.0, "san")
    b = models.Builder(ctx, t, "san", 1.0, "bf16", 5)
    x = b.input((1, 14, 14, 128))
    y = b.conv(x, 64, 3, 1, 1, act="relu")                 # per-tap-box conv
    os.environ["BLESS_TC_HALO"] = "1"
    os.environ["BLESS_TC_CFG"] = "32,64,2"
    b.conv(y, 64, 3, 1, 1, act="relu")                     # halo conv, split-K 2
    os.environ.pop("BLESS_TC_HALO")
    os.environ.pop("BLESS_TC_CFG")
    b.pool(y, 2, 2, 0, "max")
    q = b.input((128, 3 * 128))
    h = b.attention(q, 2, 64)
    g = b.gemm(h, 256, act="gelu", bias=True)
    b.layernorm(g)
    for k in range(len(b.m.layers)):
        for lo, hi in ((0, S), (8, 12)):
            ctx.run_kernel(t, k, lo, hi)
    torch.cuda.synchronize()
    print(f"{len(b.m.layers)} kernels x 2 ranges ok", flush=True)
    ctx.close()
    ctx = capi.Ctx(0, squad_max=4)
    ms = models.build_config(ctx, "C1", "fp32")
    for m in ms:
        for k in range(len(m.layers)):
            ctx.set_profile_row(m.tenant, k, [max(2000, 300000 // s) for s in range(1, S + 1)], S)
    ctx.start()
    base = capi.now_ns() + 1_000_000
    ids = [ctx.submit(j, base + i * 30_000) for i in range(2) for j in range(2)]
    ctx.drain(int(120e9))
    ctx.stop()
    assert all(ctx.poll(r)[0] == capi.BL_OK for r in ids)
    print(f"BLESS C1 run ok: {len(ctx.decisions())} squads, {len(ctx.launches())} launches", flush=True)
    ctx.close()


if __name__ == "__main__":
    main()
