# Session-4: one ncu --set full capture of the BK = 128 tcgen05 conv (VGG conv 56x56 256->256).
set -x
O=gpurun_out/s4full; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 400 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_bk128_full python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 > $O/ncu.log 2>&1
BLESS_TC_BK128=0 timeout 400 ncu --set full --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/conv_bk64_full python tools/onek.py conv 56 56 256 256 3 1 1 --launches 5 >> $O/ncu.log 2>&1
ls -la $O
