#!/bin/bash
# host-launch vs graph probe
cd $GRAFT_REPO_ROOT
O=gpurun_out/r4a; mkdir -p $O
nproc > $O/host.txt; lscpu | grep -i "model name" >> $O/host.txt
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for c in C2 C3; do timeout 600 python tools/graph_probe.py --config $c > $O/graph_probe_$c.txt 2>&1; done
cat $O/host.txt $O/graph_probe_C2.txt $O/graph_probe_C3.txt
