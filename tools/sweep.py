"""Parameter sweep of the BLESS runtime on the GPU (runs bench.py per point).

  python tools/sweep.py --config C3 --grid "split_pct=0,25,50" "squad_max=20,50"
Prints one line per point: BLESS mean, per-tenant attainment, baselines.
"""
import argparse
import itertools
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--grid", nargs="+", default=["split_pct=0,50"])
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--requests", type=int, default=60)
    ap.add_argument("--rho", default="0.5")
    ap.add_argument("--reuse-profile", action="store_true",
                    help="profile once into profiles/ and reuse it (default: every point profiles its own kernels)")
    a = ap.parse_args()
    axes = []
    for g in a.grid:
        k, vs = g.split("=")
        axes.append([(k, v) for v in vs.split(",")])
    prof = os.path.join(ROOT, "profiles", f"profile_{a.config}_b200.txt")
    if a.reuse_profile and not os.path.exists(prof):   # profile once (kernel configs are autotuned at registration), reuse for all points
        os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
        subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--config", a.config, "--no-cpu-baseline",
                        "--no-baselines", "--steps", "1", "--warmup", "1", "--requests", "10"], capture_output=True)
        for kind in ("profile", "tctune"):
            gen = os.path.join(ROOT, "gpurun_out", f"{kind}_{a.config}_rank0.txt")
            if os.path.exists(gen):
                os.makedirs(os.path.dirname(prof), exist_ok=True)
                with open(gen) as f, open(prof.replace("profile_", kind + "_"), "w") as g:
                    g.write(f.read())
    for point in itertools.product(*axes):
        args = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", a.config, "--no-cpu-baseline", "--no-slo",
                "--steps", str(a.steps), "--warmup", "1", "--requests", str(a.requests), "--also", ""]
        args += ["--rho", a.rho]
        if a.reuse_profile and os.path.exists(prof):
            args += ["--load-profile", prof]
        for k, v in point:
            args += ["--" + k.replace("_", "-"), v]
        r = subprocess.run(args, capture_output=True, text=True)
        try:
            d = json.loads(r.stdout.strip().splitlines()[-1])
        except Exception:
            print(point, "FAILED", r.stderr[-500:])
            continue
        b = d["baselines"]
        att = [round(v.get("attainment_pct", 0)) for v in d["per_tenant"].values()]
        print(" ".join(f"{k}={v}" for k, v in point), f"BLESS {d['value']:.3f} att {att} "
              f"STATIC {b['STATIC']['all_mean_ms']:.3f} Twc {b['TEMPORAL_Twc']['all_mean_ms']:.3f} "
              f"Tcap {b['TEMPORAL_Tcap']['all_mean_ms']:.3f} UNB {b['UNBOUND']['all_mean_ms']:.3f} "
              f"gap {d['scheduler']['timeline'].get('gap_us_median')}", flush=True)


if __name__ == "__main__":
    main()
