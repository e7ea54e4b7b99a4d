#!/bin/bash
# MMA rate with the halo access pattern + phase traces of the halo conv per stage split
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2x; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_bench tools/tma_bench.cu -lcuda > $O/build_bench.log 2>&1
timeout 300 /tmp/tma_bench > $O/tma_bench.txt 2>&1
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE BLESS_TC_AUTOTUNE=0 BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1
timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_tight.txt 2>&1
BLESS_TC_HALO_NA=1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_na1.txt 2>&1
BLESS_TC_HALO_KB=160 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_160.txt 2>&1
BLESS_TC_HALO_POW2=1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/trace_pow2.txt 2>&1
grep "MMA 128" $O/tma_bench.txt | tail -12
