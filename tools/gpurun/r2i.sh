#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2i; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE BLESS_TC_AUTOTUNE=0
BLESS_TC_CFG=64,128,1 timeout 300 python tools/tctrace.py conv 56 56 256 256 3 1 1 --act=relu > $O/trace_box.txt 2>&1
BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 300 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_halo64.txt 2>&1
BLESS_TC_HALO=1 BLESS_TC_CFG=32,64,1 timeout 300 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_halo32.txt 2>&1
BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,4 timeout 300 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_halo64s4.txt 2>&1
