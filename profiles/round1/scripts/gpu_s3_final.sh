# Session-3 final evidence (GPU box only): tools/gpu_evidence.sh plus the C3/C4
# ablation variants.
set -x
bash tools/gpu_evidence.sh ev_s3b
O=gpurun_out/ev_s3b
for C in C3 C4; do for a in 1 3; do
  timeout 1200 python bench.py --config $C --no-cpu-baseline --no-slo --steps 3 --ablate $a > $O/bench_${C}_ablate$a.json 2> $O/bench_${C}_ablate$a.err
done; done
ls -la $O
