# Session-3: full GPU test suite + smoke + C2 bench after the tc CTA cap (GPU box only).
set -x
O=gpurun_out/s3check; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" > $O/smoke.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
tail -1 $O/smoke.log; tail -2 $O/pytest_gpu.log
