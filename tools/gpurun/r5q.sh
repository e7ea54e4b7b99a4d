#!/bin/bash
# im2col staging: 8 loads in flight per thread vs one per loop trip
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5q; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_IM2COL_SERIAL_STAGE
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
for rep in 1 2; do timeout 600 python tools/kprobe.py --config C2 --reps 30 --only im2col > $O/base_$rep.txt 2>&1; done
unset BLESS_EXTRA_NVFLAGS
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
for rep in 1 2; do timeout 600 python tools/kprobe.py --config C2 --reps 30 --only im2col > $O/unroll_$rep.txt 2>&1; done
grep -h im2col $O/base_*.txt $O/unroll_*.txt
timeout 900 python -m pytest tests/test_gpu_c2.py tests/test_gpu_c34.py tests/test_gpu_kernels.py -q -x -k "im2col or C2 or C3 or C4 or c2 or c34" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
