#!/bin/bash
# programmatic-dependent-launch release latency (trace build)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3f; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE BLESS_TC_AUTOTUNE=0
BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/halo.txt 2>&1
timeout 600 python tools/tctrace.py gemm 128 128 64 > $O/tiny.txt 2>&1
timeout 600 python tools/tctrace.py gemm 384 1024 1024 > $O/bert.txt 2>&1
timeout 600 python tools/tctrace.py conv 7 7 512 512 3 1 1 > $O/c7.txt 2>&1
grep "event avg\|griddep\|pdl_wait\|  9 exit" $O/*.txt
