# Session-3: shared-memory-staged im2col (GPU box only): parity + kernel times.
set -x
O=gpurun_out/s3im2col; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_c2.py -q -x > $O/tests.log 2>&1
timeout 600 python tools/kprobe.py --config C2 --mode time > $O/kprobe_C2.txt 2>&1
timeout 600 python tools/kprobe.py --config C4 --mode time > $O/kprobe_C4.txt 2>&1
tail -2 $O/tests.log; grep -E "im2col" $O/kprobe_C2.txt $O/kprobe_C4.txt
