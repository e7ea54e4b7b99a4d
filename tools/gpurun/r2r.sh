#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2r; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for solo in 0 2 4 8; do for i in 1 2; do
  timeout 900 python bench.py --steps 20 --warmup 5 --also "" --no-slo --no-cpu-baseline --squad-max-solo $solo --out-dir $O/s$solo > $O/bench_solo${solo}_$i.json 2> $O/err_${solo}_$i.txt
done; done
