#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2t; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_concurrent.py tests/test_gpu_c2.py -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python tools/breakdown.py --policies BLESS,ISO > $O/breakdown.json 2> $O/err.txt
for i in 1 2; do
timeout 900 python bench.py --steps 20 --warmup 5 --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/bench_$i.json 2> $O/berr_$i.txt
done
