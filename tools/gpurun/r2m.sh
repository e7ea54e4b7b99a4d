#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2m; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python tools/breakdown.py > $O/breakdown_c2.json 2> $O/breakdown.err
