#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2j; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/kernels.log 2>&1; echo "rc=$?" >> $O/kernels.log
timeout 900 python tools/halo_ab.py > $O/halo_ab.log 2>&1
for s in "gemm 18944 256 4096" "gemm 384 4096 1024" "gemm 128 3072 768" "conv 56 56 256 256 3 1 1" "conv 14 14 256 256 3 1 1"; do
  timeout 120 python tools/onek.py $s >> $O/onek.log 2>&1
done
