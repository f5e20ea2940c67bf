#!/bin/bash
# bin-2 static item distribution A/B; ncu source-level capture of the cfg4 round kernel
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/variants.py --configs 1 4 8 --variants default tools/alt/static.so > gpurun_out/r4f_variants.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_persistent -c 1 -o gpurun_out/r4f_full_c4 -f python tools/run_once.py --config 4 --loop-mode persistent > gpurun_out/r4f_ncu.log 2>&1
