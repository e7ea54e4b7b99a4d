"""Microbenchmark: tcgen05 GEMM time vs K with a fixed tile count (one tile
per SM) to expose the per-k-block pipeline cost and the fixed per-kernel cost.

  python tools/tcsweep.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    build.build(verbose=False)
    for (M, N) in [(128 * 148, 32), (128 * 74, 64), (128 * 37, 128)]:
        for K in [64, 256, 1024, 4096]:
            ctx = capi.Ctx(0)
            S = ctx.device_info().sm_count
            t = ctx.register_tenant(1.0, "g")
            b = Builder(ctx, t, "g", 1.0, "bf16", seed=3)
            x = b.input((M, K))
            b.gemm(x, N, act="none", bias=False)
            ki = ctx.kernel_info(t, 0)
            ns, d = ctx.profile_kernel(t, 0, S, 20)
            kb = (K + 63) // 64
            print(f"M={M:6d} N={N:4d} K={K:5d} kb={kb:3d} {ki.family.decode():14s} tiles={ki.tiles:4d} "
                  f"t={ns / 1e3:7.2f}us  {ki.flops / ns / 1e3:7.1f} TF/s  {ki.bytes / ns:7.1f} GB/s")
            ctx.close()


if __name__ == "__main__":
    main()
