# Session-3: C2 load sweep rho in {0.3, 0.5, 0.7} with the final build (GPU box only).
set -x
O=gpurun_out/s3rho; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python tools/sweep.py --config C2 --steps 3 --grid "rho=0.3,0.5,0.7" > $O/c2_rho.txt 2>&1
timeout 2400 python tools/sweep.py --config C3 --steps 3 --grid "rho=0.2,0.3,0.4" > $O/c3_rho.txt 2>&1
cat $O/c2_rho.txt $O/c3_rho.txt
