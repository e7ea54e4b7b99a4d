set -x
O=gpurun_out/r1s; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for i in 1 2; do timeout 300 python tools/kprobe.py --config C2 --mode time | grep TOTAL; timeout 300 python tools/kprobe.py --config C4 --mode time | grep TOTAL; done > $O/early.txt 2>&1
cp tools/tc_gemm_lateclaim.cu paper_conf_eurosys_zhangcc0xz0g25_b200/csrc/kernels/tc_gemm.cu
python -c "import __graft_entry__ as g; g.build()" > $O/build2.log 2>&1
for i in 1 2; do timeout 300 python tools/kprobe.py --config C2 --mode time | grep TOTAL; timeout 300 python tools/kprobe.py --config C4 --mode time | grep TOTAL; done > $O/late.txt 2>&1
