"""tcgen05 GEMM pipeline microbenchmark: time vs K (one 128-row M tile per SM,
so every CTA runs exactly one tile) for several N tiles and shared-memory
pipeline budgets.  The slope over K is the per-k-block cost of the
TMA -> MMA pipeline, the intercept the fixed per-kernel cost.

  python tools/kbsweep.py                 # K sweep x BN x smem budget
  python tools/kbsweep.py --shape 384 4096 1024   # one shape x configs x budgets
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def time_gemm(M, N, K, cfg, smem_kb, reps=20):
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    os.environ["BLESS_TC_CFG"] = cfg
    os.environ["BLESS_TC_SMEM_KB"] = str(smem_kb)
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    t = ctx.register_tenant(1.0, "g")
    b = Builder(ctx, t, "g", 1.0, "bf16", seed=3)
    b.gemm(b.input((M, K)), N, act="none", bias=False)
    ki = ctx.kernel_info(t, 0)
    ns, d = ctx.profile_kernel(t, 0, S, reps)
    ctx.close()
    return ns, ki


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--shape", type=int, nargs=3)
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build
    build.build(verbose=False)
    if a.shape:
        M, N, K = a.shape
        for cfg in ["128,64,1", "64,64,1", "256,64,1", "128,64,2"]:
            for kb in [96, 128, 160, 200]:
                ns, ki = time_gemm(M, N, K, cfg, kb)
                print(f"M={M} N={N} K={K} cfg={cfg:9s} smem={kb:3d}KB tiles={ki.tiles:4d} t={ns / 1e3:7.2f}us "
                      f"{ki.flops / ns / 1e3:7.1f} TF/s", flush=True)
        return
    for BN in [64, 128, 256]:
        M = 128 * 148 if BN < 256 else 128 * 148
        N = BN
        for kb in [96, 160, 200]:
            for K in [64, 256, 512, 1024, 2048, 4096]:
                ns, ki = time_gemm(M, N, K, f"{BN},64,1", kb)
                print(f"BN={BN:3d} smem={kb:3d}KB K={K:5d} kb={K // 64:3d} tiles={ki.tiles:4d} t={ns / 1e3:7.2f}us "
                      f"{ki.flops / ns / 1e3:7.1f} TF/s {ki.bytes / ns:7.1f} GB/s", flush=True)


if __name__ == "__main__":
    main()
