#!/bin/bash
# SM-range barrier (R37): parity + barrier check, then c% x barrier sweeps on C3 / C2 / C4
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4g; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_concurrent.py -q -x -k "BLESS_range" -s > $O/pytest_range.log 2>&1; echo "pytest rc=$?"; tail -12 $O/pytest_range.log
timeout 1500 python tools/sweep.py --config C3 --grid "barrier=0,1" "split_pct=25,50,100" --steps 2 --requests 60 > $O/sweep_C3.txt 2>&1
cat $O/sweep_C3.txt
timeout 900 python tools/sweep.py --config C2 --grid "barrier=0,1" "split_pct=25,50,100" --steps 2 --requests 100 > $O/sweep_C2.txt 2>&1
cat $O/sweep_C2.txt
timeout 1500 python tools/sweep.py --config C4 --grid "barrier=0,1" "split_pct=25,100" "squad_max=10,100" --steps 2 --requests 30 > $O/sweep_C4.txt 2>&1
cat $O/sweep_C4.txt
