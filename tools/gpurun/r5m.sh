#!/bin/bash
# im2col K padding 64 vs 32 (first CNN layers): per-kernel times + parity of the first layers
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5m; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for ka in 64 32 16; do
  BLESS_IM2COL_KALIGN=$ka timeout 600 python tools/kprobe.py --config C2 --reps 30 > $O/kprobe_ka$ka.txt 2>&1
  echo "== Kalign $ka"; grep -E "^(vgg11|resnet50) +[01] " $O/kprobe_ka$ka.txt; grep TOTAL $O/kprobe_ka$ka.txt
done
for ka in 32 16; do
  BLESS_IM2COL_KALIGN=$ka timeout 900 python -m pytest tests/test_gpu_c2.py tests/test_gpu_c34.py -q -x > $O/pytest_ka$ka.log 2>&1; echo "parity Kalign $ka rc=$?"; tail -1 $O/pytest_ka$ka.log
done
