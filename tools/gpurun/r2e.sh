#!/bin/bash
# halo conv: parity (descriptor base offset on, then off if needed) + A/B timing
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2e
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > gpurun_out/r2e/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "halo" > gpurun_out/r2e/halo_bo1.log 2>&1; rc=$?
echo "rc=$rc" >> gpurun_out/r2e/halo_bo1.log
if [ $rc -ne 0 ]; then
  BLESS_EXTRA_NVFLAGS=-DBLESS_TC_HALO_BO=0 python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)" > gpurun_out/r2e/build0.log 2>&1
  timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "halo" > gpurun_out/r2e/halo_bo0.log 2>&1; echo "rc=$?" >> gpurun_out/r2e/halo_bo0.log
fi
timeout 900 python tools/halo_ab.py > gpurun_out/r2e/halo_ab.log 2>&1
