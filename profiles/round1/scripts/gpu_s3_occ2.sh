# Session-3: per-family occupancy caps -- full GPU tests, kprobe, C2/C3/C4 bench (GPU box only).
set -x
O=gpurun_out/s3occ2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
for C in C2 C3 C4; do timeout 600 python tools/kprobe.py --config $C --mode time > $O/kprobe_$C.txt 2>&1; done
timeout 900 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2.json 2> $O/bench_c2.err
timeout 900 python bench.py --config C3 --no-cpu-baseline --no-slo > $O/bench_c3.json 2> $O/bench_c3.err
timeout 1200 python bench.py --config C4 --no-cpu-baseline --no-slo > $O/bench_c4.json 2> $O/bench_c4.err
tail -3 $O/pytest_gpu.log; grep TOTAL $O/kprobe_*.txt
