#!/bin/bash
# S_max re-tune after the kernel speed-up: C2 (rho 0.5) and C3/C4 (rho 0.3, 0.5)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3i; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 --also "" --no-cpu-baseline --no-slo --out-dir $O/c2base > $O/c2base.json 2> $O/c2base.err
for sm in 40 60 80 120; do
  timeout 600 python bench.py --steps 10 --warmup 3 --also "" --no-cpu-baseline --no-baselines --load-profile $O/c2base/profile_C2_gpu0.txt \
     --squad-max $sm --out-dir $O/c2_sm$sm > $O/c2_sm$sm.json 2> $O/c2_sm$sm.err
done
for cfg in C3 C4; do for rho in 0.3 0.5; do
  b=${cfg}_r${rho}
  timeout 900 python bench.py --config $cfg --rho $rho --steps 3 --warmup 3 --also "" --no-cpu-baseline --no-slo --out-dir $O/$b > $O/$b.json 2> $O/$b.err
  for sm in 20 40 80; do
    timeout 900 python bench.py --config $cfg --rho $rho --steps 3 --warmup 3 --also "" --no-cpu-baseline --no-baselines \
       --load-profile $O/$b/profile_${cfg}_gpu0.txt --squad-max $sm --out-dir $O/${b}_sm$sm > $O/${b}_sm$sm.json 2> $O/${b}_sm$sm.err
  done
done; done
python - <<'PY'
import json, glob, os
def show(base, pat):
    b = json.load(open(base))
    iso = {k: v["mean_ms"] for k, v in b["baselines"]["ISO"].items() if isinstance(v, dict)}
    print(os.path.basename(base), "BLESS(S_max default)", round(b["value"], 4), {k: round(v["all_mean_ms"], 4) for k, v in b["baselines"].items() if isinstance(v, dict) and "all_mean_ms" in v},
          {k: round(v, 1) for k, v in b["summary"]["attainment_pct"].items()})
    for f in sorted(glob.glob(pat)):
        try:
            d = json.load(open(f))
        except Exception:
            print(f, "failed"); continue
        att = {k: round(100 * iso[k] / v["mean_ms"], 1) for k, v in d["per_tenant"].items()}
        print("   ", os.path.basename(f), round(d["value"], 4), att)
show("gpurun_out/r3i/c2base.json", "gpurun_out/r3i/c2_sm*.json")
for cfg in ("C3", "C4"):
    for rho in ("0.3", "0.5"):
        try:
            show(f"gpurun_out/r3i/{cfg}_r{rho}.json", f"gpurun_out/r3i/{cfg}_r{rho}_sm*.json")
        except Exception as e:
            print(cfg, rho, "failed", e)
PY
