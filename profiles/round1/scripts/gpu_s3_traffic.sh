# Session-3: refresh ncu DRAM traffic per kernel (C2/C3/C4) with the current
# kernels, plus one --set full capture of the dominant tc conv at its tuned
# configuration (forced, so no autotuning launches precede it) and of FC1.
set -x
O=gpurun_out/s3traffic; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for C in C2 C3 C4; do
  timeout 900 ncu --nvtx --nvtx-include "traffic/" --clock-control none --csv \
      --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
      --log-file $O/traffic_$C.csv python tools/traffic.py launch --config $C --order $O/traffic_${C}_order.json > $O/traffic_$C.log 2>&1
done
BLESS_TC_CFG=128,64,1 timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 2 -c 1 -o $O/conv4_full python tools/onek.py conv 56 56 256 256 3 1 1 --launches 4 > $O/ncu_conv4.log 2>&1
BLESS_TC_CFG=128,64,3 timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 2 -c 1 -o $O/conv6_full python tools/onek.py conv 28 28 512 512 3 1 1 --launches 4 > $O/ncu_conv6.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv -s 2 -c 1 -o $O/gemv_full python tools/onek.py gemv 4096 25088 --launches 4 > $O/ncu_gemv.log 2>&1
ls -la $O
