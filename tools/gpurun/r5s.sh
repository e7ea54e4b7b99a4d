#!/bin/bash
# C2 Semi-SP c% 25 vs 50 (paper's optimum, L410) at S_max 40, interleaved on one box
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5s; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for rep in 1 2; do for c in 25 50; do
  timeout 900 python bench.py --steps 10 --warmup 3 --split-pct $c --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/c2_c${c}_$rep.json 2> $O/c2_c${c}_$rep.err
  python - $O/c2_c${c}_$rep.json <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); s = d["summary"]
print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), "STATIC", round(s["mean_ms"]["STATIC"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()}, s["replay"])
PY
done; done
