#!/bin/bash
# uniform-datapath MMA issue: parity of every tcgen05 family + halo A/B + traces
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3a; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q > $O/parity_kernels.log 2>&1
tail -2 $O/parity_kernels.log
timeout 1500 python tools/halo_ab.py > $O/halo_ab.log 2>&1
grep BEST $O/halo_ab.log
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE BLESS_TC_AUTOTUNE=0
BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 600 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/halo_64_1.txt 2>&1
BLESS_TC_CFG=128,64,1 timeout 600 python tools/tctrace.py gemm 384 4096 1024 > $O/gemm_128_64_1.txt 2>&1
grep "issue ->\|event avg" $O/*.txt
