# Session-3: §6.8 ablation on C2 (GPU box only): full BLESS, without the
# multi-task scheduler, without the determiner, without both; even 50% quotas
# (the paper's ablation setup) and the config's 1/3-2/3.
set -x
O=gpurun_out/s3ablate; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for q in "0.5,0.5" "0.333333,0.666667"; do
  for a in 0 1 2 3; do
    timeout 600 python bench.py --no-cpu-baseline --no-slo --steps 3 --quotas $q --ablate $a > $O/b_${q}_$a.json 2> $O/b_${q}_$a.err
    python - "$O/b_${q}_$a.json" "$q" "$a" <<'PY' >> $O/ablate.txt
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
b = d["baselines"]
att = {k: round(v["attainment_pct"]) for k, v in d["per_tenant"].items()}
mean = {k: round(v["mean_ms"], 3) for k, v in d["per_tenant"].items()}
print(f"quotas {sys.argv[2]} ablate {sys.argv[3]} BLESS {d['value']:.3f} per-tenant {mean} att {att} "
      f"STATIC {b['STATIC']['all_mean_ms']:.3f} Twc {b['TEMPORAL_Twc']['all_mean_ms']:.3f} "
      f"replay {d['scheduler']['oracle_replay_bit_exact']} sp_squads {d['scheduler']['sp_squads']}/{d['scheduler']['decisions']}")
PY
  done
done
cat $O/ablate.txt
