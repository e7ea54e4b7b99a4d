# Session-4 closing evidence with BK = 128 as the default: smoke, pytest -m gpu,
# bench C2 (full) / C3 / C4, reference arm, per-kernel tables.
set -x
O=gpurun_out/${1:-s4fin}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" > $O/smoke.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
tail -n 3 $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
tail -n 1 $O/bench_c2.json | cut -c1-600
for C in C2 C3 C4; do timeout 600 python tools/kprobe.py --config $C --mode time > $O/kprobe_$C.txt 2>&1; done
timeout 900 python bench.py --config C3 --no-cpu-baseline > $O/bench_c3.json 2> $O/bench_c3.err
timeout 1200 python bench.py --config C4 --no-cpu-baseline > $O/bench_c4.json 2> $O/bench_c4.err
grep TOTAL $O/kprobe_*.txt
