# Session-3: BN = 256 tiles (one CTA per SM, 192 KB of stages) vs the tuned
# configurations on the feed-bound convs/GEMMs (GPU box only).
set -x
O=gpurun_out/s3bn256; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x > $O/kernel_tests.log 2>&1
t() { echo "cfg $1 $(BLESS_TC_CFG=$1 python tools/onek.py ${@:2} 2>&1 | tail -1)"; }
{
for c in 128,64,1 256,64,1 256,64,2 256,64,3 256,64,5; do t $c conv 56 56 256 256 3 1 1; done
for c in 128,64,3 256,64,1 256,64,3 256,64,5 256,64,9; do t $c conv 28 28 256 512 3 1 1; done
for c in 128,64,3 256,64,2 256,64,3 256,64,5 256,64,9; do t $c conv 28 28 512 512 3 1 1; done
for c in 64,64,9 256,64,4 256,64,9 256,64,18; do t $c conv 14 14 512 512 3 1 1; done
for c in 128,64,1 256,64,1 256,64,2; do t $c conv 56 56 128 256 3 1 1; done
for c in 64,64,1 256,64,1 256,64,2; do t $c conv 56 56 64 256 1 1 0; done
for c in 32,64,8 256,64,4 256,64,8; do t $c conv 7 7 512 2048 1 1 0; done
for c in 128,64,1 256,64,1 256,64,2; do t $c gemm 384 4096 1024; done
for c in 128,64,1 256,64,1 256,64,2 256,64,4; do t $c gemm 384 1024 4096; done
} > $O/bn256.txt 2>&1
# what the autotuner now picks for C2's convs
timeout 900 python bench.py --no-cpu-baseline --no-slo > $O/bench_c2.json 2> $O/bench_c2.err
tail -2 $O/kernel_tests.log; grep "^cfg" $O/bn256.txt
