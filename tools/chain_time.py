"""Isolated request latency: each tenant's whole kernel sequence as one chain
on its quota SMs and on all SMs (bl_run_squad: stamped launches, PDL, median
of reps) -- the quantity the launch cadence and per-kernel fixed costs decide.

  python tools/chain_time.py --config C2 [--reps 10]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    ms = models.build_config(ctx, a.config, "fp32" if a.config == "C1" else "bf16")
    for m in ms:
        for k in range(len(m.layers)):   # run_squad needs no profile; tenant_info needs quota SMs only
            ctx.set_profile_row(m.tenant, k, [1000] * S, S)
    env = {k: os.environ.get(k) for k in ("BLESS_CARVEOUT", "BLESS_PDL")}
    for m in ms:
        q = ctx.tenant_info(m.tenant)[0]
        n = len(m.layers)
        full, kn = ctx.run_squad([(m.tenant, k, 0, S) for k in range(n)], a.reps)
        quota, _ = ctx.run_squad([(m.tenant, k, 0, q) for k in range(n)], a.reps)
        print(f"{m.name:12s} {n:3d} kernels: chain on {S} SMs {full / 1e3:8.1f} us, on its {q} quota SMs "
              f"{quota / 1e3:8.1f} us, sum of in-chain kernel times {sum(kn) / 1e3:8.1f} us  env {env}", flush=True)
    ctx.close()


if __name__ == "__main__":
    main()
