set -x
O=gpurun_out/r1i; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "gemv" > $O/pytest_gemv.log 2>&1
for r in 8 4 2 1; do BLESS_GEMV_ROWS=$r python tools/onek.py gemv 4096 25088; BLESS_GEMV_ROWS=$r python tools/onek.py gemv 4096 4096; BLESS_GEMV_ROWS=$r python tools/onek.py gemv 1000 4096; done > $O/gemv_rows.txt 2>&1
python tools/onek.py gemv 4096 25088 >> $O/gemv_rows.txt 2>&1
for s in "gemm 384 4096 1024" "gemm 384 1024 4096" "gemm 384 3072 1024" "ln 384 1024" "attn 384 16" "conv 14 14 1024 256 1 1 0"; do python tools/onek.py $s; done > $O/onek.txt 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tc_gemm -s 3 -c 1 -o $O/ffn1 python tools/onek.py gemm 384 4096 1024 --launches 5 > $O/ncu1.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:LayerNorm -s 3 -c 1 -o $O/ln python tools/onek.py ln 384 1024 --launches 5 > $O/ncu2.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:gemv -s 3 -c 1 -o $O/gemv python tools/onek.py gemv 4096 25088 --launches 5 > $O/ncu3.log 2>&1
ls $O
