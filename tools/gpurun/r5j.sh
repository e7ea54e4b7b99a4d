#!/bin/bash
# split-K fix-up: fence + atomic + fence vs one acq_rel atomic (A/B on split-K layers), parity of the variant
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5j; mkdir -p $O
export BLESS_TC_AUTOTUNE=0
run_set() {
  for v in "1 32,64,4 conv 14 14 256 256 3 1 1" "1 32,64,8 conv 7 7 512 512 3 1 1" "0 32,64,5 conv 7 7 2048 512 1 1 0" \
           "0 32,64,9 conv 28 28 256 256 3 2 1" "1 128,64,6 conv 28 28 512 512 3 1 1" "1 32,64,1 conv 28 28 512 512 3 1 1" \
           "1 128,64,4 conv 14 14 512 512 3 1 1" "1 32,64,4 conv 14 14 512 512 3 1 1"; do
    set -- $v
    h=$1; cfg=$2; shift 2
    BLESS_TC_HALO=$h BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py "$@" --reps 50 2>&1 | tail -1 | sed "s/^/cfg=$cfg halo=$h /"
  done
}
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
echo "== baseline (fence + atomic + fence)"; run_set | tee $O/base.txt
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_SPLIT_ATOM_ACQREL
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
echo "== acq_rel atomic"; run_set | tee $O/acqrel.txt
unset BLESS_TC_AUTOTUNE
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/pytest_acqrel.log 2>&1; echo "kernel parity with acq_rel rc=$?"; tail -1 $O/pytest_acqrel.log
unset BLESS_EXTRA_NVFLAGS
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
