set -x
O=gpurun_out/r1k; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
timeout 600 python tools/kbsweep.py --shape 384 4096 1024 > $O/kbsweep_ffn1.txt 2>&1
timeout 300 python tools/kbsweep.py --shape 3136 64 576 > $O/kbsweep_r50c2.txt 2>&1
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
for s in "gemm 384 4096 1024" "conv 14 14 1024 256 1 1 0" "gemm 18944 64 64" "conv 56 56 64 64 3 1 1" "conv 7 7 512 2048 1 1 0"; do timeout 300 python tools/tctrace.py $s; done > $O/tctrace.txt 2>&1
tail -3 $O/pytest_gpu.log
