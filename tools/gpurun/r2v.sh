#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2v; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
export BLESS_TC_AUTOTUNE=0
for s in "gemm 18944 256 4096" "gemm 384 4096 1024" "gemm 384 1024 4096" "gemm 384 3072 1024" "conv 56 56 256 256 3 1 1"; do
  for kb in 96 160 200; do
    for cfg in "128,64,1" "64,128,1"; do BLESS_TC_SMEM_KB=$kb BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py $s | sed "s/^/smem$kb mt128 $cfg /" >> $O/onek.log 2>&1; done
    BLESS_TC_SMEM_KB=$kb BLESS_TC_MT=256 BLESS_TC_CFG=128,64,1 timeout 120 python tools/onek.py $s | sed "s/^/smem$kb mt256 128,64,1 /" >> $O/onek.log 2>&1
  done
done
