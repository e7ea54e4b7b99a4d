#!/bin/bash
# phase traces of ResNet50-shaped tcgen05 convs (trace build; rebuilt normally at the end)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4h; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
for sh in "56 56 64 64 3 1 1" "28 28 128 128 3 1 1" "14 14 256 256 3 1 1" "7 7 512 512 3 1 1" "56 56 64 256 1 1 0" "14 14 1024 256 1 1 0"; do
  timeout 300 python tools/tctrace.py conv $sh --act=relu >> $O/trace_resnet.txt 2>&1
done
unset BLESS_EXTRA_NVFLAGS
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
grep -E "^conv|pdl_wait|acc_ready|epi_done|exit|griddep|MMA warp|first 8" $O/trace_resnet.txt | head -80
