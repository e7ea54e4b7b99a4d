set -x
O=gpurun_out/r1o; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python tools/sweep.py --config C3 --grid "squad_max=4,6,8,10" "lookahead_us=20,200" "split_pct=25" > $O/sweep_c3b.txt 2>&1
timeout 1500 python tools/sweep.py --config C4 --grid "squad_max=6,10,20" "split_pct=25" > $O/sweep_c4.txt 2>&1
cp profiles/profile_C4_b200.txt profiles/tctune_C4_b200.txt $O/ 2>/dev/null
