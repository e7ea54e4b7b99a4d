# Session-3 closing evidence with the final code (GPU box only).
set -x
bash tools/gpu_evidence.sh ev_s3c
O=gpurun_out/ev_s3c
timeout 2400 python tools/sweep.py --config C2 --steps 3 --grid "rho=0.3,0.5,0.7" > $O/c2_rho.txt 2>&1
timeout 2400 python tools/sweep.py --config C3 --steps 3 --grid "rho=0.2,0.3,0.4" > $O/c3_rho.txt 2>&1
ls -la $O
