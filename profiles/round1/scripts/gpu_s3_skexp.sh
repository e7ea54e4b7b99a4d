# Session-3: split-K reduction experiments (GPU box only): red order rotation,
# plain stores instead of reds (timing only).
set -x
O=gpurun_out/s3skexp; mkdir -p $O
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/kernel_tests.log 2>&1
for v in "0 0" "1 0" "0 1"; do
  set -- $v
  export BLESS_TC_SK_ROT=$1 BLESS_TC_SK_EXP=$2
  for cfg in 128,64,1 128,64,2 64,64,2; do echo "rot=$1 exp=$2 cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py gemm 384 4096 1024 2>&1 | tail -1)"; done
  for cfg in 128,64,2 64,64,2; do echo "rot=$1 exp=$2 cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 56 56 256 256 3 1 1 2>&1 | tail -1)"; done
  for cfg in 32,64,4 64,64,4; do echo "rot=$1 exp=$2 cfg $cfg $(BLESS_TC_CFG=$cfg python tools/onek.py conv 14 14 512 512 3 1 1 2>&1 | tail -1)"; done
done > $O/skexp.txt 2>&1
tail -2 $O/kernel_tests.log; cat $O/skexp.txt
