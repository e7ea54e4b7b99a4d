#!/bin/bash
# residual preload before the accumulator wait: per-kernel A/B + parity
cd $GRAFT_REPO_ROOT
O=gpurun_out/r5o; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_NO_RES_PRELOAD
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
for rep in 1 2; do timeout 600 python tools/kprobe.py --config C2 --reps 30 > $O/kprobe_base_$rep.txt 2>&1; done
unset BLESS_EXTRA_NVFLAGS
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(force=True, verbose=False)"
for rep in 1 2; do timeout 600 python tools/kprobe.py --config C2 --reps 30 > $O/kprobe_pre_$rep.txt 2>&1; done
grep TOTAL $O/kprobe_*.txt
timeout 1500 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_concurrent.py tests/test_gpu_c2.py tests/test_gpu_c34.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
python - <<'PY'
import re
def load(f):
    d = {}
    for l in open(f):
        m = re.match(r"(\w+)\s+(\d+)\s+(\S+)\s+tiles=\s*\d+\s+d=\s*\d+\s+t=\s*([\d.]+)us.*\s(\S+)$", l.strip())
        if m: d[(m.group(1), int(m.group(2)))] = (m.group(3), float(m.group(4)), m.group(5))
    return d
b = [load(f"gpurun_out/r5o/kprobe_base_{i}.txt") for i in (1, 2)]
p = [load(f"gpurun_out/r5o/kprobe_pre_{i}.txt") for i in (1, 2)]
for k in b[0]:
    bb = min(x[k][1] for x in b); pp = min(x[k][1] for x in p)
    if abs(bb - pp) > 0.25: print(k, b[0][k][0], b[0][k][2], f"{bb:.2f} -> {pp:.2f}")
PY
