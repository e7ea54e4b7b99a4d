# Session-3: GEMV weight stream with an L2 evict-first policy -- C2 bench
# (BLESS / ISO / STATIC per-tenant latency), GEMV alone, GEMV parity.
set -x
O=gpurun_out/s3l2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k gemv > $O/gemv_tests.log 2>&1
python tools/onek.py gemv 4096 25088 > $O/gemv.txt 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2.json 2> $O/bench_c2.err
timeout 900 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2_b.json 2> $O/bench_c2_b.err
tail -2 $O/gemv_tests.log; cat $O/gemv.txt
