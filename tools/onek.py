"""One kernel, alone: build a single-layer tenant and time it at full GPU
(CUDA events, bl_profile_kernel), or launch it N times for an ncu capture.

  python tools/onek.py gemm 384 4096 1024            # time
  python tools/onek.py gemv 4096 25088 --launches 3  # launch 3x (ncu -k regex:gemv -s 2 -c 1)
  python tools/onek.py ln 384 1024
  python tools/onek.py conv 56 56 64 64 3 1 1
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("kind", choices=["gemm", "gemv", "ln", "conv", "attn"])
    ap.add_argument("dims", type=int, nargs="+")
    ap.add_argument("--launches", type=int, default=0, help="launch N times (no timing) for ncu")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--sms", type=int, default=0, help="run on logical SMs [0, sms) (a tenant's range; 0 = all)")
    a = ap.parse_args()
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    build.build(verbose=False)
    ctx = capi.Ctx(0)
    S = ctx.device_info().sm_count
    t = ctx.register_tenant(1.0, "k")
    b = Builder(ctx, t, "k", 1.0, "bf16", seed=7)
    d = a.dims
    if a.kind == "gemm":
        b.gemm(b.input((d[0], d[2])), d[1], act="gelu", bias=True)
    elif a.kind == "gemv":
        b.gemm(b.input((1, d[1])), d[0], act="relu", bias=True)
    elif a.kind == "ln":
        b.layernorm(b.input((d[0], d[1])))
    elif a.kind == "attn":
        b.attention(b.input((d[0], 3 * d[1] * 64)), d[1], 64)
    else:
        H, W, C, K, k, s, p = d
        b.conv(b.input((1, H, W, C)), K, k, s, p, act="relu", bn=True)
    ki = ctx.kernel_info(t, 0)
    sms = a.sms or S
    if a.launches:
        for _ in range(a.launches):
            ctx.run_kernel(t, 0, 0, sms)
        torch.cuda.synchronize()
        print(f"{ki.family.decode()} launched {a.launches}x")
        return
    ns, dd = ctx.profile_kernel(t, 0, sms, a.reps)
    print(f"{a.kind} {d} on {sms} SMs {ki.family.decode()} tiles={ki.tiles} d={dd} t={ns / 1e3:.2f}us "
          f"{ki.bytes / ns:.1f} GB/s {ki.flops / ns / 1e3:.1f} TF/s")


if __name__ == "__main__":
    main()
