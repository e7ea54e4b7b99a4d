# Round-end GPU evidence: smoke, pytest -m gpu, bench C2 (full) / C3 / C4, the
# reference (oracle) arm, an ncu launch list of one C2 step, per-kernel tables.
# Usage (from the repo root, on the GPU box): bash tools/gpu_evidence.sh <outdir-name>
set -x
OUT=${1:-ev}
O=gpurun_out/$OUT
mkdir -p $O
nproc > $O/host.txt; lscpu | head -20 >> $O/host.txt; nvidia-smi >> $O/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" > $O/smoke.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
timeout 900 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err
timeout 600 python bench.py --impl reference > $O/bench_c2_reference.json 2> $O/bench_c2_reference.err
timeout 900 python bench.py --config C3 --no-cpu-baseline > $O/bench_c3.json 2> $O/bench_c3.err
timeout 1200 python bench.py --config C4 --no-cpu-baseline > $O/bench_c4.json 2> $O/bench_c4.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file $O/launches_c2.csv python bench.py --light --steps 1 --warmup 1 --no-cpu-baseline --load-profile gpurun_out/profile_C2_rank0.txt > $O/ncu_bench.log 2>&1
for C in C2 C3 C4; do timeout 600 python tools/kprobe.py --config $C --mode time > $O/kprobe_$C.txt 2>&1; done
tail -3 $O/pytest_gpu.log
tail -1 $O/smoke.log
