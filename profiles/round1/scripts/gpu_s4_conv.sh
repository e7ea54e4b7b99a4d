# Session-4: confirm the restored tree on B200 (smoke + pytest -m gpu) and sweep
# the tcgen05 pipeline depth (BLESS_TC_SMEM_KB) on the load-bound VGG/ResNet
# implicit-GEMM convs.  GPU box only.
set -x
O=gpurun_out/s4conv; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" > $O/smoke.log 2>&1
for c in "56 56 256 256 3 1 1" "56 56 128 256 3 1 1" "28 28 256 512 3 1 1" "28 28 512 512 3 1 1" "14 14 512 512 3 1 1" "56 56 64 64 3 1 1" "28 28 128 128 3 1 1"; do
  for kb in 64 96 128 160 192 224; do
    echo "conv $c smem=$kb $(BLESS_TC_SMEM_KB=$kb timeout 120 python tools/onek.py conv $c 2>&1 | tail -1)" >> $O/smem_sweep.txt
  done
done
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
tail -3 $O/pytest_gpu.log
tail -1 $O/smoke.log
cat $O/smem_sweep.txt
