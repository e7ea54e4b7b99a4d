#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2s; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for solo in 4 1; do
timeout 900 python tools/breakdown.py --squad-max-solo $solo --policies BLESS,ISO > $O/breakdown_solo$solo.json 2> $O/err$solo.txt
done
