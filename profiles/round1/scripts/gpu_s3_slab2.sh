# Session-3: split-K with the chunk-major coalesced workspace (GPU box only).
set -x
O=gpurun_out/s3slab2; mkdir -p $O
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/kernel_tests.log 2>&1
for mode in 0 1; do
  export BLESS_TC_SK_MODE=$mode
  for cfg in 128,64,1 128,64,2 64,64,2; do echo "mode=$mode cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py gemm 384 4096 1024 2>&1 | tail -1)"; done
  for cfg in 128,64,1 128,64,2 64,64,2; do echo "mode=$mode cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 56 56 256 256 3 1 1 2>&1 | tail -1)"; done
  for cfg in 128,64,3 128,64,5; do echo "mode=$mode cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 28 28 512 512 3 1 1 2>&1 | tail -1)"; done
  for cfg in 32,64,4 64,64,8; do echo "mode=$mode cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 14 14 512 512 3 1 1 2>&1 | tail -1)"; done
  for cfg in 32,64,4 64,64,8; do echo "mode=$mode cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 7 7 512 512 3 1 1 2>&1 | tail -1)"; done
done > $O/slab.txt 2>&1
unset BLESS_TC_SK_MODE
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
BLESS_TC_SK_MODE=0 BLESS_TC_CFG=128,64,2 timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=none > $O/trace_red_ffn1.txt 2>&1
unset BLESS_EXTRA_NVFLAGS
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
tail -2 $O/kernel_tests.log; grep "^mode" $O/slab.txt | sed 's/tc_conv_bf16//; s/tc_gemm_bf16//'; grep -A16 "reps=1:" $O/trace_red_ffn1.txt
