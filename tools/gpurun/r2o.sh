#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2o; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 300 python tools/sanitize.py > $O/plain.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > $O/sanitizer_$tool.log 2>&1
  echo "rc=$?" >> $O/sanitizer_$tool.log
done
timeout 600 python -m pytest tests/test_gpu_c1.py -q -x -k steal -s > $O/steal.log 2>&1; echo "rc=$?" >> $O/steal.log
