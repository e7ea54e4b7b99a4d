# Session-4: what sets the tcgen05 kernel's ~0.5 us per K block?  Same layers
# with BK = 64 / 32 / 16 (bytes per stage halve, TMA rows per byte double).
set -x
O=gpurun_out/s4bk; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for cfg in "128,64,1" "128,32,1" "128,16,1" "64,64,1" "64,32,1"; do
  echo "cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py conv 56 56 256 256 3 1 1 2>&1 | tail -1)" >> $O/bk.txt
  echo "cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py gemm 18944 256 4096 2>&1 | tail -1)" >> $O/bk.txt
  echo "cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py gemm 384 4096 1024 2>&1 | tail -1)" >> $O/bk.txt
done
cat $O/bk.txt
