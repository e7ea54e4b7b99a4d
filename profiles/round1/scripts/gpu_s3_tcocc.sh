# Session-3: CTAs per SM of the tcgen05 kernel on unrestricted launches (GPU box only).
set -x
O=gpurun_out/s3tcocc; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for occ in 2 1; do for C in C2 C3 C4; do BLESS_TC_MAX_OCC=$occ timeout 600 python tools/kprobe.py --config $C --mode time > $O/kprobe_${C}_tc$occ.txt 2>&1; done; done
grep TOTAL $O/kprobe_*
