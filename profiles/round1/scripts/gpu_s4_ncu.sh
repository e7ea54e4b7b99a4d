# Session-4: ncu launch list of one C2 bench step with the BK = 128 kernels
# (profile table loaded, so the capture holds the step, not the profiler).
set -x
O=gpurun_out/s4ncu2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file $O/launches_c2.csv python bench.py --light --steps 1 --warmup 1 --no-cpu-baseline --load-profile profiles/profile_C2_b200.txt > $O/ncu_bench.log 2>&1
ls -la $O; tail -n 3 $O/ncu_bench.log
