#!/bin/bash
# S_max defaults: paper's 50 vs the round-1 sweep values, more steps
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4j; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 1500 python tools/sweep.py --config C2 --grid "squad_max=20,50,20,50" --steps 5 --requests 100 > $O/sweep_C2.txt 2>&1
timeout 1500 python tools/sweep.py --config C3 --grid "squad_max=10,50" --steps 3 --requests 60 > $O/sweep_C3.txt 2>&1
timeout 1800 python tools/sweep.py --config C4 --grid "squad_max=10,50,100" --steps 3 --requests 30 > $O/sweep_C4.txt 2>&1
cat $O/sweep_C2.txt $O/sweep_C3.txt $O/sweep_C4.txt
