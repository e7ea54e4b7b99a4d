# ncu dram traffic per kernel for C2/C3/C4 (tools/traffic.py), plus one full
# capture of the dominant kernels.  Usage (GPU box): bash tools/gpu_traffic.sh <outdir>
set -x
O=gpurun_out/${1:-traffic}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for C in C2 C3 C4; do
  timeout 900 ncu --nvtx --nvtx-include "traffic/" --clock-control none --csv \
      --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
      --log-file $O/traffic_$C.csv python tools/traffic.py launch --config $C --order $O/traffic_${C}_order.json > $O/traffic_$C.log 2>&1
done
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_full python tools/onek.py conv 56 56 128 256 3 1 1 --launches 5 > $O/ncu_conv.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv -s 3 -c 1 -o $O/gemv_full python tools/onek.py gemv 4096 25088 --launches 5 > $O/ncu_gemv.log 2>&1
ls -la $O
