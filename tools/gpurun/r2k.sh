#!/bin/bash
# full GPU suite + smoke + driver bench + C2 launch list + traffic + ncu full of the top conv
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2k; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
T0=$(date +%s); timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 --out-dir $O > $O/bench.json 2> $O/bench.err; echo "rc=$? wall=$(( $(date +%s) - T0 ))" >> $O/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c2.csv python bench.py --steps 1 --warmup 0 --light --requests 20 --load-profile $O/profile_C2_gpu0.txt --out-dir $O/ncu_bench > $O/launches.log 2>&1
timeout 900 ncu --nvtx --nvtx-include "traffic/" --clock-control none --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --log-file $O/traffic_C2.csv python tools/traffic.py launch --config C2 --order $O/traffic_C2_order.json > $O/traffic.log 2>&1
BLESS_TC_AUTOTUNE=0 BLESS_TC_HALO=1 BLESS_TC_CFG=64,64,1 timeout 500 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_halo_full python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 > $O/ncu_full.log 2>&1
