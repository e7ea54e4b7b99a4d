#!/bin/bash
# arrival wait vs solo-squad cap
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4c; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for v in "40 0 2 20" "40 4 2 20" "40 2 2 20" "40 8 2 20" "40 4 1 20" "40 4 2 5" "40 4 3 40"; do
  set -- $v
  timeout 900 python tools/breakdown.py --config C2 --squad-max $1 --squad-max-solo $2 --max-inflight $3 --lookahead-us $4 --requests 150 --policies BLESS > $O/bd_sm$1_solo$2_mi$3_la$4.json 2>&1
done
