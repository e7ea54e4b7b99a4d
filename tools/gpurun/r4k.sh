#!/bin/bash
# software dependency (swdep): kernel + concurrent parity, chain A/B, short bench A/B
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4k; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_concurrent.py tests/test_gpu_c2.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
for sw in 0 1; do
  BLESS_SWDEP=$sw timeout 600 python tools/graph_probe.py --config C2 > $O/chain_C2_swdep$sw.txt 2>&1
  BLESS_SWDEP=$sw timeout 600 python tools/kprobe.py --config C2 --reps 20 > $O/kprobe_C2_swdep$sw.txt 2>&1
done
grep -E "kernels on" $O/chain_C2_swdep*.txt
grep TOTAL $O/kprobe_C2_swdep*.txt
for sw in 0 1; do
  BLESS_SWDEP=$sw timeout 900 python bench.py --steps 4 --warmup 2 --also "" --no-slo --no-cpu-baseline --out-dir $O/b$sw > $O/bench_swdep$sw.json 2> $O/bench_swdep$sw.err
done
python - <<'PY'
import json
for sw in (0, 1):
    try:
        d = json.loads(open(f"gpurun_out/r4k/bench_swdep{sw}.json").read().strip().splitlines()[-1])
    except Exception as e:
        print(sw, "failed", e); continue
    s = d["summary"]
    print("swdep", sw, round(s["value_ms"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()},
          {k: round(v, 3) for k, v in s["mean_ms"].items()}, "roof", round(d["roofline"]["frac"], 4),
          d["roofline"]["event_avg_ns_per_launch"], "fallbacks", d["scheduler"]["fallback_launches"], d["scheduler"]["oracle_replay_bit_exact"])
PY
