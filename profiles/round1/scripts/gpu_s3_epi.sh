# Session-3: unsplit epilogue store A/B (GPU box only): default vs warp-staged
# full-sector stores (-DBLESS_TC_EPI_STG) vs no stores (-DBLESS_TC_NOSTORE).
set -x
O=gpurun_out/s3epi; mkdir -p $O
shapes=("gemm 384 4096 1024" "gemm 128 768 768" "conv 56 56 256 256 3 1 1" "conv 56 56 64 64 3 1 1" "conv 28 28 128 128 3 1 1" "conv 56 56 64 256 1 1 0" "conv 112 112 64 128 3 1 1")
for fl in "" "-DBLESS_TC_EPI_STG" "-DBLESS_TC_NOSTORE"; do
  BLESS_EXTRA_NVFLAGS="$fl" python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > $O/build.log 2>&1
  if [ "$fl" = "-DBLESS_TC_EPI_STG" ]; then timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/kernel_tests_stg.log 2>&1; fi
  for sh in "${shapes[@]}"; do echo "[$fl] $(python tools/onek.py $sh 2>&1 | tail -1)"; done >> $O/epi.txt
  BLESS_EXTRA_NVFLAGS="$fl -DBLESS_TC_TRACE" python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
  BLESS_EXTRA_NVFLAGS="$fl -DBLESS_TC_TRACE" timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=none > "$O/trace_ffn1_$fl.txt" 2>&1
  BLESS_EXTRA_NVFLAGS="$fl -DBLESS_TC_TRACE" timeout 300 python tools/tctrace.py conv 56 56 64 64 3 1 1 > "$O/trace_c64_$fl.txt" 2>&1
done
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
tail -2 $O/kernel_tests_stg.log; sed 's/tc_conv_bf16//; s/tc_gemm_bf16//' $O/epi.txt
for f in $O/trace_*; do echo "## $f"; grep -A13 "reps=1:" "$f" | grep -E "acc_ready|epi_done|exit|reps"; done
