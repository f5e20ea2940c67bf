#!/bin/bash
# k_dense at 64 registers (4 blocks/SM) A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 400 python tools/variants.py --configs 2 --variants default tools/alt/dm1024.so > gpurun_out/r4u_variants.txt 2>&1
