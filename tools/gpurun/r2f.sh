#!/bin/bash
# ncu --set full with source-level warp stall sampling: VGG conv 56x56 256->256,
# per-tap-box config (64,128,1) and halo (64,64,1)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2f; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
export BLESS_TC_AUTOTUNE=0
BLESS_TC_CFG=64,128,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_box python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 > $O/ncu_box.log 2>&1
BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_halo python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 > $O/ncu_halo.log 2>&1
BLESS_TC_CFG=128,64,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/gemm_big python tools/onek.py gemm 18944 256 4096 --launches 5 > $O/ncu_gemm.log 2>&1
ls -la $O
