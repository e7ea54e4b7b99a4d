#!/bin/bash
# C4 at rho 0.3: which kernel change moved BLESS vs STATIC (halo geometry / halo stages / no halo)
cd $GRAFT_REPO_ROOT
O=gpurun_out/r3c; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
run() { n=$1; shift; timeout 900 env "$@" python bench.py --config C4 --rho 0.3 --steps 3 --warmup 3 --also "" --no-cpu-baseline --out-dir $O/$n > $O/$n.json 2> $O/$n.err; }
run default X=1
run pow2 BLESS_TC_HALO_POW2=1
run na1 BLESS_TC_HALO_NA=1
run nohalo BLESS_TC_HALO=0
python - <<'PY'
import json
for n in ("default", "pow2", "na1", "nohalo"):
    try:
        d = json.load(open(f"gpurun_out/r3c/{n}.json")); s = d["summary"]
        print(n, {k: round(v, 3) for k, v in s["mean_ms"].items()}, {k: round(v, 1) for k, v in s["attainment_pct"].items()})
    except Exception as e:
        print(n, "failed", e)
PY
