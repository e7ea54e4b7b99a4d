set -x
O=gpurun_out/r1m; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2_par.json 2> $O/bench_c2_par.err
BLESS_LAUNCH_THREADS=0 timeout 600 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2_seq.json 2> $O/bench_c2_seq.err
timeout 600 python bench.py --config C3 --no-cpu-baseline --no-slo > $O/bench_c3_par.json 2> $O/bench_c3_par.err
BLESS_LAUNCH_THREADS=0 timeout 600 python bench.py --config C3 --no-cpu-baseline --no-slo > $O/bench_c3_seq.json 2> $O/bench_c3_seq.err
tail -3 $O/pytest_gpu.log
