# Session-3: phase trace of split-K units (GPU box only).
set -x
O=gpurun_out/s3sktrace; mkdir -p $O
export BLESS_EXTRA_NVFLAGS=-DBLESS_TC_TRACE
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force > $O/build.log 2>&1
for cfg in 128,64,1 128,64,2 64,64,2; do BLESS_TC_CFG=$cfg timeout 300 python tools/tctrace.py gemm 384 4096 1024 --act=none > $O/ffn1_$cfg.txt 2>&1; done
for cfg in 64,64,1 32,64,4 64,64,4; do BLESS_TC_CFG=$cfg timeout 300 python tools/tctrace.py conv 14 14 512 512 3 1 1 > $O/c8_$cfg.txt 2>&1; done
for cfg in 128,64,1 128,64,2; do BLESS_TC_CFG=$cfg timeout 300 python tools/tctrace.py conv 56 56 256 256 3 1 1 > $O/c4_$cfg.txt 2>&1; done
unset BLESS_EXTRA_NVFLAGS
python -m paper_conf_eurosys_zhangcc0xz0g25_b200.build --force >> $O/build.log 2>&1
for f in $O/*.txt; do echo "#### $f"; grep -A14 "reps=20" $f; done
