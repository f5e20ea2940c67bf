#!/bin/bash
# grid-barrier poll back-off sweep (SGR_BARSLEEP ns)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 700 python tools/variants.py --configs 1 2 3 4 --variants default tools/alt/bs0.so tools/alt/bs60.so tools/alt/bs200.so > gpurun_out/r5e_variants.txt 2>&1
