# Session-3: C2 operating-point sweep with the current kernels (GPU box only).
set -x
O=gpurun_out/s3sweep; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python tools/sweep.py --config C2 --steps 3 --grid "split_pct=0,25,50" "squad_max=10,20,50" > $O/c2.txt 2>&1
cat $O/c2.txt
