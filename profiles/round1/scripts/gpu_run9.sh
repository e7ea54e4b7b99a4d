set -x
O=gpurun_out/r1p; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q -k "tc_gemm or forced" > $O/pytest_tc.log 2>&1
timeout 1200 python tools/sweep.py --config C3 --grid "rho=0.2,0.3,0.4" "squad_max=10" "split_pct=25" > $O/sweep_c3_rho.txt 2>&1
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
for a in none gelu; do timeout 300 python tools/tctrace.py gemm 18944 64 64 --act=$a; timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=$a; done > $O/tctrace_act.txt 2>&1
export BLESS_EXTRA_NVFLAGS="-DBLESS_TC_TRACE -DBLESS_TC_NOSTORE"
for a in none; do timeout 300 python tools/tctrace.py gemm 18944 64 64 --act=$a; timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=$a; done > $O/tctrace_nostore.txt 2>&1
