# Session-3 diagnosis of the large VGG implicit-GEMM convs (tc_conv):
# standalone times, phase trace, one ncu --set full capture.  GPU box only.
set -x
O=gpurun_out/s3conv; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for c in "56 56 256 256 3 1 1" "28 28 512 512 3 1 1" "112 112 64 128 3 1 1"; do
  python tools/onek.py conv $c >> $O/onek.txt 2>&1
  for kb in 64 96 128 192; do BLESS_TC_SMEM_KB=$kb python tools/onek.py conv $c 2>&1 | sed "s/^/smem$kb /" >> $O/onek.txt; done
done
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv4_full python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 > $O/ncu_conv4.log 2>&1
BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 300 python tools/tctrace.py conv 56 56 256 256 3 1 1 --act=relu > $O/trace_conv4.txt 2>&1
BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE timeout 300 python tools/tctrace.py conv 28 28 512 512 3 1 1 --act=relu > $O/trace_conv6.txt 2>&1
ls -la $O
