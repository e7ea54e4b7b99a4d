#!/bin/bash
# R38 (arrivals join in-flight solo NSP squads): parity/barrier test, breakdown and bench A/B on C2
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5g; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_concurrent.py -q -x -k "BLESS_join or BLESS-" -s > $O/pytest_join.log 2>&1; echo "pytest rc=$?"; grep -E "passed|failed|squads" $O/pytest_join.log | tail -8
for b in 0 2; do
  timeout 900 python tools/breakdown.py --config C2 --squad-max 40 --barrier $b --requests 150 --policies BLESS > $O/bd_barrier$b.json 2>&1
done
for rep in 1 2; do for b in 0 2; do
  timeout 900 python bench.py --steps 10 --warmup 3 --barrier $b --also "" --no-slo --no-cpu-baseline --out-dir $O/b > $O/c2_barrier${b}_$rep.json 2> $O/c2_barrier${b}_$rep.err
  python - $O/c2_barrier${b}_$rep.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    s = d["summary"]; t = d["scheduler"]["timeline"]
    print(sys.argv[1].split("/")[-1], round(s["value_ms"], 3), "STATIC", round(s["mean_ms"]["STATIC"], 3), "Twc", round(s["mean_ms"]["TEMPORAL_Twc"], 3),
          "UNB", round(s["mean_ms"]["UNBOUND"], 3), {k: round(v, 1) for k, v in s["attainment_pct"].items()}, s["replay"], "viol", t.get("barrier_violations"))
except Exception as e:
    print(sys.argv[1], "failed", e, open(sys.argv[1].replace(".json", ".err")).read()[-800:])
PY
done; done
python - <<'PY'
import json
for b in (0, 2):
    try:
        d = json.load(open(f"gpurun_out/r5g/bd_barrier{b}.json"))
    except Exception as e:
        print(b, "bd failed", e); continue
    print("barrier", b, {n: {k: round(v, 1) for k, v in x.items()} for n, x in d["BLESS"].items()})
    print("   wait by state", {n: {k: (v["n"], round(v["mean_us"], 1)) for k, v in x.items()} for n, x in d["BLESS_wait_by_state"].items()})
PY
