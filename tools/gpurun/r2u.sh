#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2u; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "mt256" > $O/mt.log 2>&1; echo "rc=$?" >> $O/mt.log
export BLESS_TC_AUTOTUNE=0
for s in "gemm 18944 256 4096" "gemm 384 4096 1024" "gemm 384 1024 4096" "gemm 384 3072 1024" "gemm 128 3072 768" "gemm 128 768 3072"; do
  for cfg in "128,64,1" "128,128,1" "64,128,1"; do BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py $s | sed "s/^/mt128 $cfg /" >> $O/onek.log 2>&1; done
  for cfg in "128,64,1" "64,64,1" "128,64,2"; do BLESS_TC_MT=256 BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py $s | sed "s/^/mt256 $cfg /" >> $O/onek.log 2>&1; done
done
