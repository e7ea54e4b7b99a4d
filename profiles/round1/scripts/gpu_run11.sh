set -x
O=gpurun_out/r1r; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for i in 1 2; do python tools/onek.py ln 384 1024; python tools/onek.py ln 128 768; done > $O/ln_new.txt 2>&1
cp paper_conf_eurosys_zhangcc0xz0g25_b200/csrc/kernels/executor.cuh /tmp/exec_new.cuh
cp tools/executor_old.cuh paper_conf_eurosys_zhangcc0xz0g25_b200/csrc/kernels/executor.cuh
python -c "import __graft_entry__ as g; g.build()" > $O/build2.log 2>&1
for i in 1 2; do python tools/onek.py ln 384 1024; python tools/onek.py ln 128 768; done > $O/ln_old.txt 2>&1
cp /tmp/exec_new.cuh paper_conf_eurosys_zhangcc0xz0g25_b200/csrc/kernels/executor.cuh
