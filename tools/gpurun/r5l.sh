#!/bin/bash
# software dependency with a release-add count: parity, chain times, bench A/B
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5l; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
BLESS_SWDEP=1 timeout 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_concurrent.py -q -x > $O/pytest_swdep1.log 2>&1; echo "pytest swdep1 rc=$?"; tail -1 $O/pytest_swdep1.log
for sw in 0 1; do
  BLESS_SWDEP=$sw timeout 600 python tools/graph_probe.py --config C2 > $O/chain_C2_swdep$sw.txt 2>&1
  BLESS_SWDEP=$sw timeout 600 python tools/kprobe.py --config C2 --reps 20 > $O/kprobe_C2_swdep$sw.txt 2>&1
done
grep -E "kernels on" $O/chain_C2_swdep*.txt; grep TOTAL $O/kprobe_C2_swdep*.txt
for rep in 1 2; do for sw in 0 1; do
  BLESS_SWDEP=$sw timeout 900 python bench.py --steps 8 --warmup 3 --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/bench_swdep${sw}_$rep.json 2> $O/bench_swdep${sw}_$rep.err
  python - $O/bench_swdep${sw}_$rep.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    s = d["summary"]
    print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), {k: round(v, 3) for k, v in s["mean_ms"].items()}, {k: round(v, 1) for k, v in s["attainment_pct"].items()}, s["replay"], "fb", d["scheduler"]["fallback_launches"])
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done; done
