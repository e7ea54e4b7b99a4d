# Session-4: is the implicit-GEMM conv's A load slowed by the OOB columns of a
# power-of-two BW box over a non-power-of-two OW?  Same C/K, OW = 56 vs 64, 28 vs 32.
set -x
O=gpurun_out/s4oob; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for c in "56 56 256 256 3 1 1" "64 64 256 256 3 1 1" "28 28 512 512 3 1 1" "32 32 512 512 3 1 1" "56 56 256 256 1 1 0" "64 64 256 256 1 1 0"; do
  for cfg in "128,64,1" "64,64,1"; do
    echo "cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py conv $c 2>&1 | tail -1)" >> $O/oob.txt
  done
done
cat $O/oob.txt
