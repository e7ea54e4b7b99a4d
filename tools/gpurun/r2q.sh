#!/bin/bash
cd $GRAFT_REPO_ROOT
O=gpurun_out/r2q; mkdir -p $O
python -c "from paper_conf_eurosys_zhangcc0xz0g25_b200 import build; build.build(verbose=False)" > $O/build.log 2>&1
for cfg in C2 C3; do
  timeout 600 python tools/chain_time.py --config $cfg >> $O/chain.txt 2>&1
  BLESS_CARVEOUT=100 timeout 600 python tools/chain_time.py --config $cfg >> $O/chain.txt 2>&1
  BLESS_PDL=0 timeout 600 python tools/chain_time.py --config $cfg >> $O/chain.txt 2>&1
done
