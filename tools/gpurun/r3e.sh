#!/bin/bash
# 256-bit epilogue stores / residual loads: parity + epilogue trace
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3e; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q > $O/parity_kernels.log 2>&1
tail -2 $O/parity_kernels.log
export BLESS_TC_AUTOTUNE=0
BLESS_TC_CFG=128,64,1 BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 600 python tools/tctrace.py gemm 384 4096 1024 --act=gelu > $O/gelu.txt 2>&1
BLESS_TC_CFG=128,64,1 BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 600 python tools/tctrace.py gemm 384 4096 1024 --act=none > $O/none.txt 2>&1
for f in gelu none; do echo "== $f"; grep -A12 "reps=20" $O/$f.txt | grep "event avg\|acc_ready\|epi_done\|exit"; done
