#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2g
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_bench tools/tma_bench.cu -lcuda > gpurun_out/r2g/build.log 2>&1
timeout 300 /tmp/tma_bench > gpurun_out/r2g/tma_bench.txt 2>&1
