"""Microbenchmark of the tcgen05 GEMM/conv kernel's tile configurations on the
layer shapes of the configs (full GPU, CUDA events via bl_profile_kernel).

  python tools/tcsweep.py              # default config vs every forced (BN, BK, splits)
  python tools/tcsweep.py --quick      # default config only

Forcing uses BLESS_TC_CFG="BN,BK,splits", read when a kernel is appended.
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# (name, kind, dims): conv (H, W, C, K, k, stride, pad) / gemm (M, N, K)
SHAPES = [
    ("vgg.c2 112x112 64->128 3x3", "conv", (112, 112, 64, 128, 3, 1, 1)),
    ("vgg.c3 56x56 128->256 3x3", "conv", (56, 56, 128, 256, 3, 1, 1)),
    ("vgg.c4 56x56 256->256 3x3", "conv", (56, 56, 256, 256, 3, 1, 1)),
    ("vgg.c5 28x28 256->512 3x3", "conv", (28, 28, 256, 512, 3, 1, 1)),
    ("vgg.c6 28x28 512->512 3x3", "conv", (28, 28, 512, 512, 3, 1, 1)),
    ("vgg.c8 14x14 512->512 3x3", "conv", (14, 14, 512, 512, 3, 1, 1)),
    ("r50 56x56 64->64 3x3", "conv", (56, 56, 64, 64, 3, 1, 1)),
    ("r50 56x56 64->256 1x1", "conv", (56, 56, 64, 256, 1, 1, 0)),
    ("r50 56x56 256->64 1x1", "conv", (56, 56, 256, 64, 1, 1, 0)),
    ("r50 28x28 128->128 3x3", "conv", (28, 28, 128, 128, 3, 1, 1)),
    ("r50 56x56 128->128 3x3 s2", "conv", (56, 56, 128, 128, 3, 2, 1)),
    ("r50 28x28 512->128 1x1", "conv", (28, 28, 512, 128, 1, 1, 0)),
    ("r50 14x14 256->256 3x3", "conv", (14, 14, 256, 256, 3, 1, 1)),
    ("r50 14x14 1024->256 1x1", "conv", (14, 14, 1024, 256, 1, 1, 0)),
    ("r50 14x14 256->1024 1x1", "conv", (14, 14, 256, 1024, 1, 1, 0)),
    ("r50 7x7 512->512 3x3", "conv", (7, 7, 512, 512, 3, 1, 1)),
    ("r50 7x7 2048->512 1x1", "conv", (7, 7, 2048, 512, 1, 1, 0)),
    ("r50 7x7 512->2048 1x1", "conv", (7, 7, 512, 2048, 1, 1, 0)),
    ("bert-b qkv 128x2304x768", "gemm", (128, 2304, 768)),
    ("bert-b ffn1 128x3072x768", "gemm", (128, 3072, 768)),
    ("bert-b ffn2 128x768x3072", "gemm", (128, 768, 3072)),
    ("bert-l qkv 384x3072x1024", "gemm", (384, 3072, 1024)),
    ("bert-l proj 384x1024x1024", "gemm", (384, 1024, 1024)),
    ("bert-l ffn1 384x4096x1024", "gemm", (384, 4096, 1024)),
    ("bert-l ffn2 384x1024x4096", "gemm", (384, 1024, 4096)),
]

CFGS = [(bn, bk, s) for bn in (32, 64, 128, 256) for bk in (64, 32) for s in (1, 2, 3, 4, 6, 8)
        if not (bk == 32 and bn < 256)]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--filter", default="")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    build.build(verbose=False)
    for name, kind, dims in SHAPES:
        if a.filter and a.filter not in name:
            continue
        ctx = capi.Ctx(0)
        S = ctx.device_info().sm_count
        t = ctx.register_tenant(1.0, "g")
        b = Builder(ctx, t, "g", 1.0, "bf16", seed=3)
        cfgs = [None] + ([] if a.quick else CFGS)
        if kind == "conv":
            H, W, C, K, k, s, p = dims
            x = b.input((1, H, W, C))
        else:
            M, N, K = dims
            x = b.input((M, K))
        res = []
        for cfg in cfgs:
            if cfg is None:
                os.environ.pop("BLESS_TC_CFG", None)
            else:
                os.environ["BLESS_TC_CFG"] = ",".join(map(str, cfg))
            if kind == "conv":
                b.conv(x, K, k, s, p, act="relu", bn=True)
            else:
                b.gemm(x, N, act="none", bias=True)
            kid = len(b.m.layers) - 1
            ki = ctx.kernel_info(t, kid)
            ns, _ = ctx.profile_kernel(t, kid, S, a.reps)
            res.append((ns, cfg, ki.tiles, ki.flops))
        os.environ.pop("BLESS_TC_CFG", None)
        d = res[0]
        best = min(res, key=lambda r: r[0])
        line = (f"{name:30s} default {d[0] / 1e3:7.2f}us tiles={d[2]:4d} {d[3] / d[0] / 1e3:6.0f} TF/s | "
                f"best {best[0] / 1e3:7.2f}us cfg={best[1]} tiles={best[2]} {best[3] / best[0] / 1e3:6.0f} TF/s")
        print(line, flush=True)
        if not a.quick:
            top = sorted(res[1:], key=lambda r: r[0])[:6]
            print("    " + "  ".join(f"{r[1]}:{r[0] / 1e3:.1f}" for r in top), flush=True)
        ctx.close()


if __name__ == "__main__":
    main()
