#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2y; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_bench tools/tma_bench.cu -lcuda > $O/build_bench.log 2>&1
timeout 300 /tmp/tma_bench > $O/tma_bench.txt 2>&1
grep "MMA 128" $O/tma_bench.txt | tail -8
