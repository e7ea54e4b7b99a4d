#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2a/smi.txt 2>&1
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > gpurun_out/r2a/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x -s -k "concurrent or io_slo or c1 or c2" > gpurun_out/r2a/pytest_new.log 2>&1
echo "rc=$?" >> gpurun_out/r2a/pytest_new.log
