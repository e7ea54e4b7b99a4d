#!/bin/bash
# S_max x c% sweep on C2/C3/C4 with the current kernels (each point profiles itself)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4d; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 1500 python tools/sweep.py --config C3 --grid "squad_max=10,20,50,100" "split_pct=25,50" --steps 2 --requests 60 > $O/sweep_C3.txt 2>&1
timeout 1500 python tools/sweep.py --config C4 --grid "squad_max=10,20,50,100" "split_pct=25,50" --steps 2 --requests 30 > $O/sweep_C4.txt 2>&1
timeout 900 python tools/sweep.py --config C2 --grid "squad_max=20,40,57,100" "split_pct=25,50" --steps 2 --requests 100 > $O/sweep_C2.txt 2>&1
cat $O/sweep_C3.txt $O/sweep_C4.txt $O/sweep_C2.txt
