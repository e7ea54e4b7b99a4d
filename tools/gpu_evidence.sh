# Round-end GPU evidence: smoke, pytest -m gpu, bench C2/C3/C4, ncu launch list.
# Usage (from the repo root, on the GPU box): bash tools/gpu_evidence.sh <outdir-name>
set -x
OUT=${1:-ev}
mkdir -p gpurun_out/$OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" > gpurun_out/$OUT/smoke.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/$OUT/pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/$OUT/bench_c2.json 2> gpurun_out/$OUT/bench_c2.err
timeout 600 python bench.py --config C3 --no-cpu-baseline > gpurun_out/$OUT/bench_c3.json 2> gpurun_out/$OUT/bench_c3.err
timeout 900 python bench.py --config C4 --no-cpu-baseline > gpurun_out/$OUT/bench_c4.json 2> gpurun_out/$OUT/bench_c4.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/$OUT/launches_c2.csv python bench.py --light --steps 1 --warmup 1 --no-cpu-baseline --load-profile gpurun_out/profile_C2_rank0.txt > gpurun_out/$OUT/ncu_bench.log 2>&1
tail -3 gpurun_out/$OUT/pytest_gpu.log
tail -1 gpurun_out/$OUT/smoke.log
