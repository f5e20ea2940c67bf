#!/bin/bash
# where the warps spend their time on cfg4 / cfg3 (phase-cycle build)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
SGR_PHASES=1 SGR_LIBPATH=tools/alt/pc.so timeout 600 python tools/bin_cycles.py 4 3 1 > gpurun_out/r4e_cycles.txt 2>&1
