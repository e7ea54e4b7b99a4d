#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4i; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python bench.py --config C3 --steps 1 --warmup 1 --requests 60 --also "" --no-slo --no-cpu-baseline --no-baselines --dump-squads 400 --out-dir $O > $O/bench_C3.json 2> $O/bench_C3.err
tail -2 $O/bench_C3.err
