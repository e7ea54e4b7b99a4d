# Session-3: split-K epilogue cost (GPU box only).  A/B of the semaphore fence
# (one fence per unit vs every thread) over forced (BN, BK, splits) configs,
# plus the phase trace of one split configuration.
set -x
O=gpurun_out/s3splitk; mkdir -p $O
run() {
  for cfg in 128,64,1 128,64,2 64,64,2 32,64,4; do echo "cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py gemm 384 4096 1024 2>&1 | tail -1)"; done
  for cfg in 64,64,1 64,64,2 128,64,2 128,64,3; do echo "cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 56 56 256 256 3 1 1 2>&1 | tail -1)"; done
  for cfg in 128,64,1 128,64,3 128,64,5 64,64,3; do echo "cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 28 28 512 512 3 1 1 2>&1 | tail -1)"; done
  for cfg in 64,64,1 32,64,4 64,64,4 128,64,9; do echo "cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 14 14 512 512 3 1 1 2>&1 | tail -1)"; done
  for cfg in 32,64,1 32,64,4 64,64,4; do echo "cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 14 14 256 256 3 1 1 2>&1 | tail -1)"; done
}
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > $O/build.log 2>&1
run > $O/one_fence.txt 2>&1
BLESS_EXTRA_NVFLAGS=-DBLESS_TC_SPLIT_FENCE_ALL python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
run > $O/fence_all.txt 2>&1
BLESS_TC_CFG=128,64,2 BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=none > $O/trace_split2.txt 2>&1
BLESS_TC_CFG=128,64,1 BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=none > $O/trace_split1.txt 2>&1
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/kernel_tests.log 2>&1
tail -3 $O/kernel_tests.log
paste $O/one_fence.txt $O/fence_all.txt | cut -c1-400
