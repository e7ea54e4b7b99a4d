#!/bin/bash
# ncu --set full of the two dominant tcgen05 families with the bench's tuned configs (no autotune
# candidates), on all SMs and on the tenant's quota range; the stats-ring wrap test
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5b; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_c1.py -q -x -k "ring or replay" -s > $O/pytest_ring.log 2>&1; echo "pytest rc=$?"; grep -E "passed|failed|launches," $O/pytest_ring.log | tail -3
export BLESS_TC_AUTOTUNE=0
for sms in 0 49; do
  BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv3x3_vgg_56x56x256_sms$sms python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 --sms $sms > $O/ncu_vgg_$sms.log 2>&1
  BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 python tools/onek.py conv 56 56 256 256 3 1 1 --sms $sms >> $O/onek_times.txt 2>&1
done
for sms in 0 99; do
  BLESS_TC_HALO=0 BLESS_TC_CFG=64,64,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv1x1_r50_14x14x1024x256_sms$sms python tools/onek.py conv 14 14 1024 256 1 1 0 --launches 5 --sms $sms > $O/ncu_r50_$sms.log 2>&1
  BLESS_TC_HALO=0 BLESS_TC_CFG=64,64,1 python tools/onek.py conv 14 14 1024 256 1 1 0 --sms $sms >> $O/onek_times.txt 2>&1
done
cat $O/onek_times.txt
