#!/bin/bash
# C3 diagnosis: bench line (timeline, prediction errors) + breakdown
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4e; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python bench.py --config C3 --steps 2 --warmup 1 --requests 60 --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/bench_C3.json 2> $O/bench_C3.err
timeout 900 python tools/breakdown.py --config C3 --squad-max 20 --requests 60 --policies BLESS,STATIC,UNBOUND > $O/bd_C3.json 2>&1
