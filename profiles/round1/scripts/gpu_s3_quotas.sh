# Session-3: Table 2 two-model quota sets + biased workload E on C2 (GPU box only).
set -x
O=gpurun_out/s3quotas; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 3000 python tools/quota_sweep.py --steps 3 > $O/quotas.txt 2>&1
cat $O/quotas.txt
