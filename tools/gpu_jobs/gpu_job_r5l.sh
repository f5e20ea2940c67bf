#!/bin/bash
# GS huge-member threshold sweep (512 / 2048 default / 8192)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for lib in default tools/alt/gs512.so tools/alt/gs8k.so; do if [ $lib = default ]; then timeout 300 python tools/gs_quick.py; else SGR_LIBPATH=$lib timeout 300 python tools/gs_quick.py; fi; done > gpurun_out/r5l_gs.txt 2>&1
