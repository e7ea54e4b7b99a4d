#!/bin/bash
# epilogue cost: GELU vs no activation vs no stores (trace build, BERT-large ffn1 shape)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3d; mkdir -p $O
export BLESS_TC_AUTOTUNE=0 BLESS_TC_CFG=128,64,1
BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 600 python tools/tctrace.py gemm 384 4096 1024 --act=gelu > $O/gelu.txt 2>&1
BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 600 python tools/tctrace.py gemm 384 4096 1024 --act=none > $O/none.txt 2>&1
BLESS_EXTRA_NVFLAGS="-DBLESS_TC_TRACE -DBLESS_TC_NOSTORE" timeout 600 python tools/tctrace.py gemm 384 4096 1024 --act=gelu > $O/gelu_nostore.txt 2>&1
for f in gelu none gelu_nostore; do echo "== $f"; grep -A12 "reps=20" $O/$f.txt | grep "event avg\|acc_ready\|epi_done\|exit"; done
