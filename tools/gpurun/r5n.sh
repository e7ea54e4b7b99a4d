#!/bin/bash
# final evidence: acq_rel split-K fix-up + im2col K 32: full GPU suite, smoke, bench x3, launch list
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5n; mkdir -p $O
nproc > $O/host.txt; lscpu | grep -i "model name" >> $O/host.txt
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
tail -2 $O/smoke.log
for i in 1 2 3; do
  T0=$(date +%s); timeout 1800 python bench.py --gpus 1 --steps 20 --warmup 5 --out-dir $O/run$i > $O/bench_$i.json 2> $O/bench_$i.err; echo "rc=$? wall=$(( $(date +%s) - T0 ))" >> $O/bench_$i.err
  tail -1 $O/bench_$i.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c2.csv python bench.py --steps 1 --warmup 0 --light --requests 20 --load-profile $O/run1/profile_C2_gpu0.txt --out-dir $O/ncu_bench > $O/launches.log 2>&1
python - <<'PY'
import json
for i in (1, 2, 3):
    try:
        d = json.loads(open(f"gpurun_out/r5n/bench_{i}.json").read().strip().splitlines()[-1])
    except Exception as e:
        print("bench", i, "failed", e); continue
    s = d["summary"]
    print(i, round(s["value_ms"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()},
          {k: round(v, 3) for k, v in s["mean_ms"].items()}, "roof", d["roofline"]["kernel"], round(d["roofline"]["frac"], 4), s["replay"])
    print("  ", json.dumps(s.get("other_configs")))
PY
