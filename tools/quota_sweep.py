"""PAPER.md Table 2 (L295) two-model quota sets and workload E (biased load,
L298) on config C2 (VGG11 + ResNet50), one bench.py run per point (GPU box).

  python tools/quota_sweep.py [--steps 3]
Prints one line per point: quotas, per-tenant rho, BLESS mean, per-tenant
attainment %, and the STATIC / TEMPORAL / UNBOUND means on the same traces.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# (VGG11 quota, ResNet50 quota): the seven two-model sets of Table 2
SETS = [(1 / 3, 2 / 3), (7 / 18, 11 / 18), (4 / 9, 5 / 9), (1 / 2, 1 / 2), (5 / 9, 4 / 9), (11 / 18, 7 / 18),
        (2 / 3, 1 / 3)]
# workload E: ResNet50 provisions 8/9 of the GPU at low load, the other app 1/9 at high load
BIASED = ((1 / 9, 8 / 9), (0.9, 0.2))


def run(quotas, rhos, steps):
    args = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", "C2", "--no-cpu-baseline", "--no-slo", "--also", "",
            "--steps", str(steps), "--warmup", "3", "--quotas", ",".join(f"{q:.6f}" for q in quotas)]
    if rhos:
        args += ["--rhos", ",".join(str(r) for r in rhos)]
    r = subprocess.run(args, capture_output=True, text=True)
    try:
        d = json.loads(r.stdout.strip().splitlines()[-1])
    except Exception:
        print(quotas, "FAILED", r.stderr[-400:], flush=True)
        return
    b = d["baselines"]
    att = {k: round(v["attainment_pct"]) for k, v in d["per_tenant"].items()}
    qs = {k: v["quota_sms"] for k, v in d["per_tenant"].items()}
    print(f"quotas {[round(q, 3) for q in quotas]} sms {qs} rho {rhos or 0.5} BLESS {d['value']:.3f} att {att} "
          f"STATIC {b['STATIC']['all_mean_ms']:.3f} Twc {b['TEMPORAL_Twc']['all_mean_ms']:.3f} "
          f"Tcap {b['TEMPORAL_Tcap']['all_mean_ms']:.3f} UNB {b['UNBOUND']['all_mean_ms']:.3f}", flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=3)
    a = ap.parse_args()
    for q in SETS:
        run(q, None, a.steps)
    run(BIASED[0], BIASED[1], a.steps)


if __name__ == "__main__":
    main()
