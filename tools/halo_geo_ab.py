"""A/B of the halo conv's tile geometry and stage split (B200): power-of-two
tile width (round 2's first halo kernel: BW = 64 for OW = 56, one 34 KB halo
stage + 3 weight stages in 113 KB) against the tight width BW = OW + 2 (a 31 KB
halo stage, so two halo stages + two weight stages fit), plus a forced single
halo stage and a 160 KB budget.  Each variant: every halo tile configuration,
CUDA-event timing (bl_profile_kernel, back to back with PDL, weights L2-warm),
and a max-relative-error check of the output against torch's fp32 conv.

  python tools/halo_geo_ab.py [--reps 20]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SHAPES = [(112, 112, 64, 128), (56, 56, 128, 256), (56, 56, 256, 256), (28, 28, 256, 512), (28, 28, 512, 512),
          (14, 14, 512, 512), (56, 56, 64, 64), (28, 28, 128, 128), (14, 14, 256, 256), (7, 7, 512, 512)]
VARIANTS = [("pow2", {"BLESS_TC_HALO_POW2": "1"}), ("tight", {}), ("tight_na1", {"BLESS_TC_HALO_NA": "1"}),
            ("tight_160KB", {"BLESS_TC_HALO_KB": "160"})]
CFGS = ["32,64,1", "64,64,1", "128,64,1", "32,64,2", "64,64,2", "128,64,2", "32,64,4", "64,64,4", "128,64,4"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    import torch

    from paper_conf_eurosys_zhangcc0xz0g25_b200 import build, capi
    from paper_conf_eurosys_zhangcc0xz0g25_b200.models import Builder
    build.build(verbose=False)
    os.environ["BLESS_TC_AUTOTUNE"] = "0"
    os.environ["BLESS_TC_HALO"] = "1"
    for H, W, C, K in SHAPES:
        best = {}
        for vname, env in VARIANTS:
            for k in ("BLESS_TC_HALO_POW2", "BLESS_TC_HALO_NA", "BLESS_TC_HALO_KB"):
                os.environ.pop(k, None)
            os.environ.update(env)
            for cfg in CFGS:
                os.environ["BLESS_TC_CFG"] = cfg
                ctx = capi.Ctx(0)
                S = ctx.device_info().sm_count
                t = ctx.register_tenant(1.0, "k")
                b = Builder(ctx, t, "k", 1.0, "bf16", seed=3)
                x = b.input((1, H, W, C))
                y = b.conv(x, K, 3, 1, 1, act="relu", bn=True)
                ki = ctx.kernel_info(t, 0)
                if ki.family.decode() != "tc_conv_bf16":
                    ctx.close()
                    continue
                ns, d = ctx.profile_kernel(t, 0, S, a.reps)
                ctx.run_kernel(t, 0)
                torch.cuda.synchronize()
                L = b.m.layers[-1]
                w = L.w.float().reshape(K, 3, 3, C).permute(0, 3, 1, 2)
                ref = torch.nn.functional.conv2d(x.float().permute(0, 3, 1, 2), w, padding=1)
                ref = torch.relu(ref * L.scale.view(1, -1, 1, 1) + L.shift.view(1, -1, 1, 1)).permute(0, 2, 3, 1)
                err = float(((y.float() - ref).abs().max() / ref.abs().max().clamp_min(1e-6)))
                print(f"conv {H}x{W} {C}->{K} {vname:11s} cfg={cfg:9s} tiles={ki.tiles:4d} smem={ki.smem // 1024:3d}KB "
                      f"t={ns / 1e3:7.2f}us {ki.flops / ns / 1e3:6.1f} TF/s err={err:.1e}", flush=True)
                if vname not in best or ns < best[vname][0]:
                    best[vname] = (ns, cfg)
                ctx.close()
        print(f"BEST conv {H}x{W} {C}->{K}: " + ", ".join(f"{v} {ns / 1e3:.2f}us ({c})" for v, (ns, c) in best.items()),
              flush=True)


if __name__ == "__main__":
    main()
