#!/bin/bash
# final-code check: full GPU suite + smoke + one bench run
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5i; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 1800 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench rc=$?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/r5i/bench_default.json").read().strip().splitlines()[-1])
s = d["summary"]
print(round(s["value_ms"], 3), d["steps"], d["warmup"], {k: round(v, 1) for k, v in s["attainment_pct"].items()}, {k: round(v, 3) for k, v in s["mean_ms"].items()}, s["replay"], d["roofline"]["kernel"], round(d["roofline"]["frac"], 4))
PY
