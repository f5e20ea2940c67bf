#!/bin/bash
# hub-build knob re-check on the final kernel: bin-1 batch 16, bin-2 batch QB=4, push buffer 128
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 700 python tools/variants.py --configs 4 8 --variants default tools/alt/b1b16.so tools/alt/qb4.so tools/alt/pb128.so > gpurun_out/r5m_variants.txt 2>&1
