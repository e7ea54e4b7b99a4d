# Session-3: attention softmax over 8 warps (key halves) -- parity + timing (GPU box only).
set -x
O=gpurun_out/s3attn; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 timeout 500 python -m pytest tests/test_gpu_kernels.py -q -x -k attention > $O/tests.log 2>&1
timeout 600 python -m pytest tests/test_gpu_c34.py -q -x > $O/tests_c34.log 2>&1
for C in C3 C4; do timeout 600 python tools/kprobe.py --config $C --mode time > $O/kprobe_$C.txt 2>&1; done
tail -2 $O/tests.log $O/tests_c34.log; grep -E "attention" $O/kprobe_C4.txt | head -3; grep TOTAL $O/kprobe_*.txt
