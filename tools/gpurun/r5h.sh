#!/bin/bash
# plumbing check of the multi-GPU paths on one GPU (BLESS_BENCH_DEVICE=0): torchrun 2 ranks and one process with 2 contexts
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5h; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
BLESS_BENCH_DEVICE=0 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --steps 2 --warmup 1 --no-cpu-baseline --no-slo --also "" --out-dir $O/tr > $O/torchrun2.json 2> $O/torchrun2.err; echo "torchrun rc=$?"
BLESS_BENCH_DEVICE=0 timeout 900 python bench.py --gpus 2 --steps 2 --warmup 1 --no-cpu-baseline --no-slo --also "" --out-dir $O/one > $O/oneproc2.json 2> $O/oneproc2.err; echo "one-process rc=$?"
BLESS_BENCH_DEVICE=0 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29612 bench.py --impl reference --gpus 2 --steps 3 --warmup 3 > $O/ref2.json 2> $O/ref2.err; echo "reference rc=$?"
for f in torchrun2 oneproc2 ref2; do echo "== $f"; tail -c 700 $O/$f.json; echo; tail -3 $O/$f.err; done
