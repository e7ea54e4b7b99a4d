#!/bin/bash
# f1 squad study (C2, C3) + the new run_squad test
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2c
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > gpurun_out/r2c/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_io_slo_temporal.py -q -x -s > gpurun_out/r2c/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2c/pytest.log
timeout 1200 python tools/squad_study.py --config C2 --squads 40 --out gpurun_out/r2c/f1_c2.json > gpurun_out/r2c/f1_c2.log 2>&1
timeout 1200 python tools/squad_study.py --config C3 --squads 30 --out gpurun_out/r2c/f1_c3.json > gpurun_out/r2c/f1_c3.log 2>&1
