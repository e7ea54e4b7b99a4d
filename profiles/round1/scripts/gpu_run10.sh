set -x
O=gpurun_out/r1q; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_c2.py -x -q > $O/pytest_k.log 2>&1
timeout 300 python tools/kprobe.py --config C2 --mode time > $O/kprobe_c2.txt 2>&1
timeout 300 python tools/kprobe.py --config C4 --mode time > $O/kprobe_c4.txt 2>&1
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
for a in none; do timeout 300 python tools/tctrace.py gemm 18944 64 64 --act=$a; timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=$a; done > $O/tctrace_co.txt 2>&1
timeout 300 python tools/tctrace.py conv 56 56 64 64 3 1 1 >> $O/tctrace_co.txt 2>&1
