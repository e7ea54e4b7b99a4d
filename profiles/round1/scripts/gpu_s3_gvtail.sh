# Session-3: GEMV split tail (last-wave row tiles cut into K halves) -- parity and A/B (GPU box only).
set -x
O=gpurun_out/s3gvtail; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k gemv > $O/tests.log 2>&1
for sh in "4096 25088" "4096 4096" "1000 4096" "1000 2048"; do
  for v in 1 0; do echo "split_tail=$v $(BLESS_GEMV_SPLIT_TAIL=$v python tools/onek.py gemv $sh 2>&1 | tail -1)"; done
done > $O/ab.txt 2>&1
tail -2 $O/tests.log; cat $O/ab.txt
