# Session-4: BK = 128 stages (one TMA box = two 64-deep SW128 slabs per operand)
# against BK = 64 on the conv/GEMM layers; parity of the BK 128 path.
set -x
O=gpurun_out/s4bk128; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q -k "tc_forced" > $O/pytest_forced.log 2>&1
BLESS_TC_BK128=1 timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q -k "tc_gemm or conv_bf16 or tc_forced" > $O/pytest_bk128.log 2>&1
tail -3 $O/pytest_forced.log $O/pytest_bk128.log
for c in "conv 56 56 256 256 3 1 1" "conv 56 56 128 256 3 1 1" "conv 28 28 512 512 3 1 1" "conv 28 28 256 512 3 1 1" "conv 14 14 512 512 3 1 1" "conv 14 14 256 256 3 1 1" "conv 56 56 256 64 1 1 0" "conv 14 14 1024 256 1 1 0" "gemm 384 4096 1024" "gemm 384 1024 4096" "gemm 128 3072 768" "gemm 18944 256 4096"; do
  for cfg in "128,64,1" "128,128,1" "64,64,1" "64,128,1"; do
    echo "cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py $c 2>&1 | tail -1)" >> $O/bk128.txt
  done
done
cat $O/bk128.txt
