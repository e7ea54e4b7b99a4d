#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2n; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for v in "20 2 20" "20 1 20" "20 1 60" "10 2 20" "10 1 20" "5 2 20" "50 2 20"; do
  set -- $v
  echo "== S_max=$1 inflight=$2 lookahead=$3" >> $O/sweep.txt
  timeout 600 python tools/breakdown.py --squad-max $1 --max-inflight $2 --lookahead-us $3 --policies BLESS,ISO >> $O/sweep.txt 2>> $O/err.txt
done
