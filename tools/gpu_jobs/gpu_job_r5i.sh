#!/bin/bash
# dense threshold re-sweep with the staged-ahead dense passes
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 500 python tools/variants.py --configs 2 --variants default tools/alt/dd4b.so tools/alt/dd16b.so tools/alt/dd32b.so > gpurun_out/r5i_variants.txt 2>&1
