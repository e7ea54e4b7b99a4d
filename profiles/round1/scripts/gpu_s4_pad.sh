# Session-4: the implicit-GEMM conv pays ~0.53 us per K block at BK = 64/32/16
# alike (s4bk).  Is it the out-of-bounds (padding) part of the 4-D TMA box?
# Same 56x56 output: pad 1 on a 56x56 input vs pad 0 on a 58x58 input.
set -x
O=gpurun_out/s4pad; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for cfg in "128,64,1" "128,16,1"; do
  for c in "56 56 256 256 3 1 1" "58 58 256 256 3 1 0" "30 30 512 512 3 1 0" "28 28 512 512 3 1 1"; do
    echo "cfg=$cfg $(BLESS_TC_CFG=$cfg timeout 120 python tools/onek.py conv $c 2>&1 | tail -1)" >> $O/pad.txt
  done
done
cat $O/pad.txt
