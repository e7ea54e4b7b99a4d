#!/bin/bash
# C3: Semi-SP c = 0 and the no-determiner ablation (always NSP) vs the default
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5e; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for rho in 0.5 0.3; do for v in "25 0" "0 0" "25 2"; do
  set -- $v
  timeout 900 python bench.py --config C3 --rho $rho --split-pct $1 --ablate $2 --steps 3 --warmup 1 --requests 80 --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/C3_rho${rho}_c$1_ab$2.json 2> $O/C3_rho${rho}_c$1_ab$2.err
  python - $O/C3_rho${rho}_c$1_ab$2.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    s = d["summary"]; t = d["scheduler"]["timeline"]
    print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), "STATIC", round(s["mean_ms"]["STATIC"], 3), "UNB", round(s["mean_ms"]["UNBOUND"], 3),
          {k: round(v, 1) for k, v in s["attainment_pct"].items()}, "busy", round(t.get("in_squad_sm_busy_frac") or 0, 3), "sp", d["scheduler"]["sp_squads"], "/", d["scheduler"]["decisions"])
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done; done
