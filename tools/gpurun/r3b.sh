#!/bin/bash
# bench with the uniform-issue kernels (x2) + chain times
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3b; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for i in 1 2; do
  timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out-dir $O/run$i > $O/bench_$i.json 2> $O/bench_$i.err
done
timeout 600 python tools/chain_time.py --config C2 > $O/chain_c2.txt 2>&1
timeout 600 python tools/chain_time.py --config C3 > $O/chain_c3.txt 2>&1
timeout 600 python tools/chain_time.py --config C4 > $O/chain_c4.txt 2>&1
python - <<'PY'
import json
for i in (1, 2):
    try:
        d = json.load(open(f"gpurun_out/r3b/bench_{i}.json"))
    except Exception as e:
        print("bench", i, "failed", e); continue
    s = d["summary"]
    print(i, round(s["value_ms"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()},
          {k: round(v, 3) for k, v in s["mean_ms"].items()}, "roof", round(d["roofline"]["frac"], 4),
          d["roofline"]["event_avg_ns_per_launch"], s.get("other_configs"))
PY
cat $O/chain_c*.txt
