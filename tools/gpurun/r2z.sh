#!/bin/bash
# per-stage event log of the halo conv (and per-tap conv) under the trace build
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2z; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE BLESS_TC_AUTOTUNE=0
BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/halo_64_1.txt 2>&1
BLESS_TC_HALO=1 BLESS_TC_CFG=128,64,2 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/halo_128_2.txt 2>&1
BLESS_TC_HALO=1 BLESS_TC_CFG=128,64,1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/halo_128_1.txt 2>&1
BLESS_TC_HALO=0 BLESS_TC_CFG=64,128,1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/tap_64_128_1.txt 2>&1
BLESS_TC_CFG=128,64,1 timeout 600 python tools/tctrace.py gemm 384 4096 1024 > $O/gemm_128_64_1.txt 2>&1
grep "issue ->" $O/*.txt
