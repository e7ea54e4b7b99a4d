#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2h
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > gpurun_out/r2h/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "halo" > gpurun_out/r2h/halo.log 2>&1; echo "rc=$?" >> gpurun_out/r2h/halo.log
timeout 900 python tools/halo_ab.py > gpurun_out/r2h/halo_ab.log 2>&1
