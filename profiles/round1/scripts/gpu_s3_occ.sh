# Session-3: blocks-per-SM cap for the SIMT executor kernels (GPU box only).
set -x
O=gpurun_out/s3occ; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for cap in 8 4 2 1; do
  for C in C2 C3 C4; do BLESS_MAX_OCC=$cap timeout 600 python tools/kprobe.py --config $C --mode time > $O/kprobe_${C}_occ$cap.txt 2>&1; done
done
for C in C2 C3 C4; do grep TOTAL $O/kprobe_${C}_occ*.txt; done
