# Session-4: which part of the 3x3 conv's K loop costs ~0.53 us per K block?
# Debug builds dropping the A loads / B loads / MMAs, at BK = 16 and 64.
set -x
O=gpurun_out/s4ab; mkdir -p $O
for fl in "" "-DBLESS_TC_SKIP_A" "-DBLESS_TC_SKIP_B" "-DBLESS_TC_SKIP_A -DBLESS_TC_SKIP_B" "-DBLESS_TC_SKIP_MMA" "-DBLESS_TC_SKIP_A -DBLESS_TC_SKIP_B -DBLESS_TC_SKIP_MMA"; do
  BLESS_EXTRA_NVFLAGS="$fl" python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > /dev/null 2>&1
  for cfg in "128,16,1" "128,64,1"; do
    echo "flags=[$fl] cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py conv 56 56 256 256 3 1 1 2>&1 | tail -1)" >> $O/ab.txt
    echo "flags=[$fl] cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py gemm 384 4096 1024 2>&1 | tail -1)" >> $O/ab.txt
  done
done
cat $O/ab.txt
