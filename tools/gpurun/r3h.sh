#!/bin/bash
# C2 scheduler knobs after the kernel speed-up: max in-flight squads x lookahead x S_max (10 steps each, same seeds)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3h; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 --also "" --no-cpu-baseline --out-dir $O/base > $O/base.json 2> $O/base.err
P=$O/base/profile_C2_gpu0.txt
for mi in 1 2 3; do for la in 5 20 60; do for sm in 10 20 40; do
  n=mi${mi}_la${la}_sm${sm}
  timeout 600 python bench.py --steps 10 --warmup 3 --also "" --no-cpu-baseline --no-baselines --load-profile $P \
     --max-inflight $mi --lookahead-us $la --squad-max $sm --out-dir $O/$n > $O/$n.json 2> $O/$n.err
done; done; done
python - <<'PY'
import json, glob, os
base = json.load(open("gpurun_out/r3h/base.json"))
iso = {k: v["mean_ms"] for k, v in base["baselines"]["ISO"].items() if isinstance(v, dict)}
print("base", round(base["value"], 4), {k: round(v["all_mean_ms"], 4) for k, v in base["baselines"].items() if isinstance(v, dict) and "all_mean_ms" in v})
rows = []
for f in sorted(glob.glob("gpurun_out/r3h/mi*.json")):
    try:
        d = json.load(open(f))
    except Exception:
        continue
    att = {k: round(100 * iso[k] / v["mean_ms"], 1) for k, v in d["per_tenant"].items()}
    rows.append((d["value"], os.path.basename(f), att))
for r in sorted(rows):
    print(round(r[0], 4), r[1], r[2])
PY
