#!/bin/bash
# latency breakdown (queueing vs service) at S_max 20 / 40 / 80
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4b; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
echo "build rc=$?"
for sm in 20 40 80; do
  timeout 900 python tools/breakdown.py --config C2 --squad-max $sm --requests 150 > $O/breakdown_sm$sm.json 2> $O/breakdown_sm$sm.err
  echo "sm $sm rc=$?"; tail -3 $O/breakdown_sm$sm.err
done
timeout 900 python tools/breakdown.py --config C2 --squad-max 40 --split-pct 50 --requests 150 --policies BLESS > $O/breakdown_sm40_c50.json 2> $O/breakdown_sm40_c50.err
