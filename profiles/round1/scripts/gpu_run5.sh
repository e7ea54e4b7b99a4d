set -x
O=gpurun_out/r1l; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q > $O/pytest_kernels.log 2>&1
timeout 300 python tools/kprobe.py --config C2 --mode time > $O/kprobe_c2.txt 2>&1
timeout 300 python tools/kprobe.py --config C4 --mode time > $O/kprobe_c4.txt 2>&1
timeout 300 python tools/kbsweep.py --shape 384 4096 1024 > $O/kbsweep_ffn1.txt 2>&1
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
for s in "gemm 384 4096 1024" "gemm 18944 64 64" "conv 56 56 64 64 3 1 1" "conv 14 14 1024 256 1 1 0"; do timeout 300 python tools/tctrace.py $s; done > $O/tctrace.txt 2>&1
tail -3 $O/pytest_kernels.log
