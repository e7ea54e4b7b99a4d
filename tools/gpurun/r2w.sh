#!/bin/bash
# tight halo geometry: parity + A/B sweep
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2w; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "halo" > $O/parity.log 2>&1
tail -3 $O/parity.log
timeout 1500 python tools/halo_geo_ab.py > $O/ab.log 2>&1
grep BEST $O/ab.log
