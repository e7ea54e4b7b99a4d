set -x
O=gpurun_out/r1n; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python tools/sweep.py --config C3 --grid "split_pct=0,25,50,100" "squad_max=10,20,50" > $O/sweep_c3.txt 2>&1
cp profiles/profile_C3_b200.txt profiles/tctune_C3_b200.txt $O/ 2>/dev/null
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
for a in none relu gelu; do timeout 300 python tools/tctrace.py gemm 18944 64 64 --act=$a; timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=$a; done > $O/tctrace_act.txt 2>&1
