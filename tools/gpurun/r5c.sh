#!/bin/bash
# S_max 10 vs 50 on C3 / C4 in the bench's other_configs setting (80 requests per tenant, seeds 1-3), same box
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5c; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for c in C3 C4; do for rho in 0.3 0.5; do for sm in 10 50; do
  timeout 900 python bench.py --config $c --rho $rho --squad-max $sm --steps 3 --warmup 1 --requests 80 --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/${c}_rho${rho}_sm$sm.json 2> $O/${c}_rho${rho}_sm$sm.err
  python - $O/${c}_rho${rho}_sm$sm.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    s = d["summary"]
    print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), "STATIC", round(s["mean_ms"]["STATIC"], 3), "Twc", round(s["mean_ms"]["TEMPORAL_Twc"], 3),
          "UNB", round(s["mean_ms"]["UNBOUND"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()})
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done; done; done
