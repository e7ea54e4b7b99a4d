set -x
O=gpurun_out/r1t; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1
timeout 1200 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
timeout 300 python tools/kprobe.py --config C2 --mode time > $O/kprobe_c2.txt 2>&1
timeout 300 python tools/kprobe.py --config C4 --mode time > $O/kprobe_c4.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2.json 2> $O/bench_c2.err
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
timeout 300 python tools/tctrace.py gemm 18944 64 64 --act=none > $O/tctrace.txt 2>&1
timeout 300 python tools/tctrace.py conv 56 56 64 64 3 1 1 >> $O/tctrace.txt 2>&1
