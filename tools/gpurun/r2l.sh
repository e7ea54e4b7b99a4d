#!/bin/bash
# bench with measured tau (3 runs for variance) + the GPU suite
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2l; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for i in 1 2; do
  timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out-dir $O --also "" > $O/bench_$i.json 2> $O/bench_$i.err
done
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
