"""Kernel probe: build a config's tenants and time every kernel at full GPU
with CUDA events (bl_profile_kernel), or run each once (for ncu captures).

  python tools/kprobe.py --config C2 --mode time     # table of per-kernel times
  python tools/kprobe.py --config C2 --mode once     # each kernel launched once (ncu)
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--mode", default="time", choices=["time", "once"])
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--only", default="", help="substring filter on family")
    a = ap.parse_args()
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    if a.mode == "time":
        for v, nm in [(0, "empty kernel"), (1, "gate+queue+exit"), (2, "gate+queue+exit+stamps"),
                      (3, "gate+queue+exit+stamps, PDL")]:
            print(f"overhead {nm:32s} {ctx.debug_overhead(v, 500) / 1e3:7.2f} us/launch (device), "
                  f"{ctx.debug_overhead(v | 4, 500) / 1e3:7.2f} us/launch call (host)")
    ms = models.build_config(ctx, a.config, "fp32" if a.config == "C1" else "bf16")
    tot = {}
    for m in ms:
        for k in range(len(m.layers)):
            ki = ctx.kernel_info(m.tenant, k)
            fam = ki.family.decode()
            if a.only and a.only not in fam:
                continue
            if a.mode == "once":
                ctx.run_kernel(m.tenant, k, 0, S)
                continue
            ns, d = ctx.profile_kernel(m.tenant, k, S, a.reps)
            tot[m.name] = tot.get(m.name, 0) + ns
            gbs = ki.bytes / ns
            tfs = ki.flops / ns / 1e3
            print(f"{m.name:9s} {k:3d} {fam:18s} tiles={ki.tiles:5d} d={d:3d} t={ns / 1e3:8.1f}us "
                  f"{gbs:8.1f} GB/s {tfs:7.1f} TF/s  {m.layers[k].name}")
    torch.cuda.synchronize()
    for n, v in tot.items():
        print(f"TOTAL {n}: {v / 1e3:.1f} us")


if __name__ == "__main__":
    main()
