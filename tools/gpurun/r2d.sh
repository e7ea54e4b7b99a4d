#!/bin/bash
# f4 sweeps: multi-app quota sets, SM-count sweep, deployment admission
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2d
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > gpurun_out/r2d/build.log 2>&1
timeout 1200 python tools/f4_sweeps.py deploy --out gpurun_out/r2d/f4_deploy.json > gpurun_out/r2d/deploy.log 2>&1
timeout 1500 python tools/f4_sweeps.py multiapp --out gpurun_out/r2d/f4_multiapp.json > gpurun_out/r2d/multiapp.log 2>&1
timeout 1500 python tools/f4_sweeps.py smsweep --out gpurun_out/r2d/f4_smsweep.json > gpurun_out/r2d/smsweep.log 2>&1
