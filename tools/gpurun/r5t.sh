#!/bin/bash
# reading R6 (seed every active request first) on vs off: C3 and C2
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5t; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for v in "C3 0.5" "C3 0.3" "C2 0.5"; do set -- $v; for sa in 1 0; do
  timeout 900 python bench.py --config $1 --rho $2 --seed-all $sa --steps 4 --warmup 2 --requests 80 --also "" --no-slo --no-cpu-baseline --no-baselines --out-dir $O/b > $O/$1_rho$2_seed$sa.json 2> $O/$1_rho$2_seed$sa.err
  python - $O/$1_rho$2_seed$sa.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); s = d["summary"]; t = d["scheduler"]["timeline"]
    print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), {k: round(v["mean_ms"], 3) for k, v in d["per_tenant"].items()}, s["replay"],
          "parts/squad", round(t["participants_per_squad_mean"], 2), "picks", round(t["picks_per_squad_mean"], 1), "busy", round(t["in_squad_sm_busy_frac"], 3))
except Exception as e:
    print(sys.argv[1], "failed", e, open(sys.argv[1].replace(".json", ".err")).read()[-600:])
PY
done; done
