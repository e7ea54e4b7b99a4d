# Session-3 experiments (GPU box only): guided GEMV tiles; tc_gemm operand-load
# ablations (debug builds that drop the A loads, the B loads or the MMAs).
set -x
O=gpurun_out/s3exp; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k gemv > $O/gemv_tests.log 2>&1
for sh in "4096 25088" "4096 4096" "1000 4096" "1000 2048"; do
  python tools/onek.py gemv $sh | sed "s/^/guided /" >> $O/gemv.txt 2>&1
  BLESS_GEMV_GUIDED=0 python tools/onek.py gemv $sh | sed "s/^/uniform /" >> $O/gemv.txt 2>&1
done
for fl in "" "-DBLESS_TC_SKIP_A" "-DBLESS_TC_SKIP_B" "-DBLESS_TC_SKIP_MMA" "-DBLESS_TC_SKIP_A -DBLESS_TC_SKIP_B" "-DBLESS_TC_SKIP_MMA -DBLESS_TC_SKIP_B"; do
  BLESS_EXTRA_NVFLAGS="$fl" python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > /dev/null 2>&1
  for cfg in "128,64,1" "64,64,1"; do
    echo "== flags [$fl] cfg $cfg" >> $O/tcab.txt
    BLESS_TC_CFG=$cfg python tools/onek.py conv 56 56 256 256 3 1 1 >> $O/tcab.txt 2>&1
    BLESS_TC_CFG=$cfg python tools/onek.py conv 28 28 512 512 3 1 1 >> $O/tcab.txt 2>&1
    BLESS_TC_CFG=$cfg python tools/onek.py gemm 384 4096 1024 >> $O/tcab.txt 2>&1
    BLESS_TC_CFG=$cfg python tools/onek.py gemm 18944 256 4096 >> $O/tcab.txt 2>&1
  done
done
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > /dev/null 2>&1
cat $O/gemv.txt $O/tcab.txt
