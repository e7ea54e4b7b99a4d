#!/bin/bash
# evidence run: full GPU suite + smoke + bench x3 + C2 launch list + traffic C2/C3/C4 + ncu full of the halo conv
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3g; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
tail -2 $O/smoke.log
for i in 1 2 3; do
  T0=$(date +%s); timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out-dir $O/run$i > $O/bench_$i.json 2> $O/bench_$i.err; echo "rc=$? wall=$(( $(date +%s) - T0 ))" >> $O/bench_$i.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c2.csv python bench.py --steps 1 --warmup 0 --light --requests 20 --load-profile $O/run1/profile_C2_gpu0.txt --out-dir $O/ncu_bench > $O/launches.log 2>&1
for c in C2 C3 C4; do
  timeout 900 ncu --nvtx --nvtx-include "traffic/" --clock-control none --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --log-file $O/traffic_$c.csv python tools/traffic.py launch --config $c --order $O/traffic_${c}_order.json > $O/traffic_$c.log 2>&1
done
BLESS_TC_AUTOTUNE=0 BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_halo_full python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 > $O/ncu_full.log 2>&1
python - <<'PY'
import json
for i in (1, 2, 3):
    try:
        d = json.load(open(f"gpurun_out/r3g/bench_{i}.json"))
    except Exception as e:
        print("bench", i, "failed", e); continue
    s = d["summary"]
    print(i, round(s["value_ms"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()},
          {k: round(v, 3) for k, v in s["mean_ms"].items()}, "roof", round(d["roofline"]["frac"], 4), d["scheduler"]["oracle_replay_bit_exact"])
    print("  ", json.dumps(s.get("other_configs")))
PY
