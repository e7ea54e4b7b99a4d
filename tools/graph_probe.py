"""Is a request chain bound by the host's launch calls?  Each tenant's whole
kernel sequence launched on its stream (as the engine does) vs the same chain
captured into one CUDA graph (bl_debug_chain), on all SMs and on the quota
SMs; plus the executor skeleton's per-launch cost stream vs graph
(bl_debug_overhead variant | 8).

  python tools/graph_probe.py --config C2 [--reps 5]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi, models
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    for v, nm in [(0, "empty kernel"), (1, "gate+queue+exit"), (3, "gate+queue+exit+stamps, PDL")]:
        dev = ctx.debug_overhead(v, 500) / 1e3
        host = ctx.debug_overhead(v | 4, 500) / 1e3
        gdev = ctx.debug_overhead(v | 8, 500) / 1e3
        ghost = ctx.debug_overhead(v | 12, 500) / 1e3
        print(f"overhead {nm:30s} stream: {dev:6.2f} us/launch device, {host:6.2f} host | "
              f"graph: {gdev:6.2f} us/launch device, graph launch call {ghost * 500:7.1f} us total", flush=True)
    ms = models.build_config(ctx, a.config, "fp32" if a.config == "C1" else "bf16")
    for m in ms:
        for k in range(len(m.layers)):
            ctx.set_profile_row(m.tenant, k, [1000] * S, S)
    for m in ms:
        q = ctx.tenant_info(m.tenant)[0]
        n = len(m.layers)
        for lo, hi, tag in [(0, S, f"all {S}"), (0, q, f"quota {q}")]:
            sd, sh = ctx.debug_chain(m.tenant, lo, hi, 0, a.reps)
            gd, gh = ctx.debug_chain(m.tenant, lo, hi, 1, a.reps)
            print(f"{m.name:12s} {n:3d} kernels on {tag:9s}: stream {sd / 1e3:8.1f} us (host enqueue {sh / 1e3:7.1f} us"
                  f" = {sh / n / 1e3:4.2f}/kernel) | graph {gd / 1e3:8.1f} us (launch call {gh / 1e3:5.1f} us)"
                  f"  graph/stream {gd / sd:5.3f}", flush=True)
    ctx.close()


if __name__ == "__main__":
    main()
