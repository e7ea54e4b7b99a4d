#!/bin/bash
# C3: in-flight squad depth x S_max
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5u; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for rho in 0.5 0.3; do for v in "2 50" "3 50" "4 50" "3 100"; do set -- $v
  timeout 900 python bench.py --config C3 --rho $rho --max-inflight $1 --squad-max $2 --steps 4 --warmup 2 --requests 80 --also "" --no-slo --no-cpu-baseline --no-baselines --out-dir $O/b > $O/C3_rho${rho}_mi$1_sm$2.json 2> $O/C3_rho${rho}_mi$1_sm$2.err
  python - $O/C3_rho${rho}_mi$1_sm$2.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); t = d["scheduler"]["timeline"]
    print(sys.argv[1].split("/")[-1], round(d["value"], 3), {k: round(v["mean_ms"], 3) for k, v in d["per_tenant"].items()}, d["scheduler"]["oracle_replay_bit_exact"], "busy", round(t["in_squad_sm_busy_frac"], 3))
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done; done
