#!/bin/bash
# smoke + the driver's bench command + the full GPU suite
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2b
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > gpurun_out/r2b/build.log 2>&1
#timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2b/smoke.log
T0=$(date +%s); timeout 1500 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2b/bench.json 2> gpurun_out/r2b/bench.err; echo "rc=$?" >> gpurun_out/r2b/bench.err
#timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r2b/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r2b/pytest.log
echo "wall=$(( $(date +%s) - T0 ))" >> gpurun_out/r2b/bench.err
