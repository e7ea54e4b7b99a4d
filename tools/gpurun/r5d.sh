#!/bin/bash
# C2: measured tau (R35) and S_max 20 vs 40, interleaved on one box
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5d; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for rep in 1 2; do
  for v in "0 20" "1 20" "0 40" "1 40"; do
    set -- $v
    BLESS_MEASURED_TAU=$1 timeout 900 python bench.py --steps 10 --warmup 3 --squad-max $2 --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/c2_tau$1_sm$2_$rep.json 2> $O/c2_tau$1_sm$2_$rep.err
    python - $O/c2_tau$1_sm$2_$rep.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    s = d["summary"]
    print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), "STATIC", round(s["mean_ms"]["STATIC"], 3), "Twc", round(s["mean_ms"]["TEMPORAL_Twc"], 3),
          "UNB", round(s["mean_ms"]["UNBOUND"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()}, s["replay"])
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
  done
done
