"""A/B of the halo implicit-GEMM 3x3 conv (one input box per 64-channel chunk
serves all nine taps) against the per-tap-box conv, per layer shape and tile
configuration, all S SMs, CUDA-event timing (bl_profile_kernel, back to back
with PDL as inside a request).

  python tools/halo_ab.py [--reps 20]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SHAPES = [  # H, W, C, K  (VGG11/16 and ResNet50 stride-1 3x3 convs)
    (112, 112, 64, 128), (56, 56, 128, 256), (56, 56, 256, 256), (28, 28, 256, 512), (28, 28, 512, 512),
    (14, 14, 512, 512), (56, 56, 64, 64), (28, 28, 128, 128), (14, 14, 256, 256), (7, 7, 512, 512),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    build.build(verbose=False)
    S = 148
    for H, W, C, K in SHAPES:
        best = {}
        for halo in (0, 1):
            cfgs = ["", "128,64,4", "32,64,1", "64,64,1", "128,64,1", "32,64,2", "64,64,2", "128,64,2", "32,64,4", "64,64,4", "64,128,1",
                    "64,128,2"]
            for cfg in cfgs:
                if halo and cfg.endswith(",128,1") or (halo and ",128," in cfg):
                    continue
                os.environ["BLESS_TC_HALO"] = str(halo)
                if cfg:
                    os.environ["BLESS_TC_CFG"] = cfg
                else:
                    os.environ.pop("BLESS_TC_CFG", None)
                os.environ["BLESS_TC_AUTOTUNE"] = "0"
                ctx = capi.Ctx(0)
                S = ctx.device_info().sm_count
                t = ctx.register_tenant(1.0, "k")
                b = Builder(ctx, t, "k", 1.0, "bf16", seed=3)
                b.conv(b.input((1, H, W, C)), K, 3, 1, 1, act="relu", bn=True)
                ki = ctx.kernel_info(t, 0)
                ns, d = ctx.profile_kernel(t, 0, S, a.reps)
                tf = ki.flops / ns / 1e3
                print(f"conv {H}x{W} {C}->{K} halo={halo} cfg={cfg or 'default':9s} tiles={ki.tiles:4d} d={d:3d} "
                      f"smem={ki.smem // 1024:3d}KB t={ns / 1e3:7.2f}us {tf:6.1f} TF/s", flush=True)
                key = "halo" if halo else "box"
                if key not in best or ns < best[key][0]:
                    best[key] = (ns, cfg)
                ctx.close()
        print(f"BEST conv {H}x{W} {C}->{K}: per-tap boxes {best['box'][0] / 1e3:.2f}us ({best['box'][1]}), "
              f"halo {best['halo'][0] / 1e3:.2f}us ({best['halo'][1]}), speedup {best['box'][0] / best['halo'][0]:.2f}x",
              flush=True)


if __name__ == "__main__":
    main()
