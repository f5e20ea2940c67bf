#!/bin/bash
# dense-pass threshold sweep (|W| > n/DIV) on the stencil; k_dense ncu; cfg2 round profile
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/variants.py --configs 2 --variants default tools/alt/dd3.so tools/alt/dd4.so tools/alt/dd8.so > gpurun_out/r4n_variants.txt 2>&1
timeout 300 python tools/round_profile_persistent.py --config 2 --every 20 > gpurun_out/r4n_rounds_c2.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_dense -c 1 -o gpurun_out/r4n_dense_c2 -f python tools/run_once.py --config 2 --loop-mode persistent > gpurun_out/r4n_ncu.log 2>&1
