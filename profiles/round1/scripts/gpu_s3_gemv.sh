# Session-3: stream-mode GEMV parity + tile-size sweep (GPU box only).
set -x
O=gpurun_out/s3gemv; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k gemv > $O/tests.log 2>&1
for sh in "4096 25088" "4096 4096" "1000 4096" "1000 2048"; do
  BLESS_GEMV_MODE=rows python tools/onek.py gemv $sh | sed "s/^/rows /" >> $O/sweep.txt 2>&1
  for ts in 1 2 4 8; do BLESS_GEMV_TILE_STAGES=$ts python tools/onek.py gemv $sh | sed "s/^/ts$ts /" >> $O/sweep.txt 2>&1; done
done
cat $O/sweep.txt
