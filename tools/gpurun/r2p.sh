#!/bin/bash
# final evidence: driver bench x3, Table-2 quota sets, f1 study with the current kernels
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2p; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for i in 1 2 3; do
  timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out-dir $O/run$i > $O/bench_$i.json 2> $O/bench_$i.err
done
timeout 1500 python tools/quota_sweep.py --steps 5 > $O/quota_sets.txt 2>&1
timeout 1200 python tools/squad_study.py --config C2 --squads 40 --out $O/f1_c2.json > $O/f1_c2.log 2>&1
