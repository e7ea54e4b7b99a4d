#!/bin/bash
# headline-style bench lines for C3 and C4 (and C1), committed code
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5p; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for c in C3 C4 C1; do for rho in 0.3 0.5; do
  timeout 1500 python bench.py --config $c --rho $rho --steps 10 --warmup 3 --also "" --no-cpu-baseline --out-dir $O/b > $O/bench_${c}_rho$rho.json 2> $O/bench_${c}_rho$rho.err; echo "$c rho $rho rc=$?"
  python - $O/bench_${c}_rho$rho.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    s = d["summary"]
    print("  ", round(s["value_ms"], 3), {k: round(v, 3) for k, v in s["mean_ms"].items()}, {k: round(v, 1) for k, v in s["attainment_pct"].items()}, s["replay"], d["roofline"]["kernel"], round(d["roofline"]["frac"], 3))
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done; done
