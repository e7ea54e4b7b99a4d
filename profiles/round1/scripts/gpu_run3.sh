set -x
O=gpurun_out/r1j; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1
timeout 300 python tools/kprobe.py --config C2 --mode time > $O/kprobe_c2.txt 2>&1
timeout 300 python tools/kprobe.py --config C4 --mode time > $O/kprobe_c4.txt 2>&1
timeout 600 python tools/kbsweep.py > $O/kbsweep.txt 2>&1
timeout 300 python tools/kbsweep.py --shape 384 4096 1024 > $O/kbsweep_ffn1.txt 2>&1
timeout 300 python tools/kbsweep.py --shape 3136 64 576 > $O/kbsweep_r50c2.txt 2>&1
tail -3 $O/pytest_gpu.log
