#!/bin/bash
# C3 squad shape at S_max 20 / 50 (no baselines)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4f; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for sm in 20 50; do
timeout 900 python bench.py --config C3 --steps 2 --warmup 1 --requests 60 --squad-max $sm --also "" --no-slo --no-cpu-baseline --no-baselines --out-dir $O/b > $O/bench_C3_sm$sm.json 2> $O/bench_C3_sm$sm.err
done
timeout 900 python bench.py --config C2 --steps 2 --warmup 1 --requests 100 --also "" --no-slo --no-cpu-baseline --no-baselines --out-dir $O/b > $O/bench_C2.json 2> $O/bench_C2.err
