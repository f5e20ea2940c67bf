#!/bin/bash
# flat build: thread-per-vertex bin 0 on ER / stencil; per-round profile of cfg2 and cfg3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/variants.py --configs 2 3 6 --variants default tools/alt/b0t.so > gpurun_out/r4i_variants.txt 2>&1
timeout 300 python tools/round_profile_persistent.py --config 2 --every 10 > gpurun_out/r4i_rounds_c2.txt 2>&1
timeout 300 python tools/round_profile_persistent.py --config 3 --every 1 > gpurun_out/r4i_rounds_c3.txt 2>&1
