#!/bin/bash
# gather throughput vs warps per SM (16.7 M u16 / int colors, random)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for b in 1 2 3 4 8; do ./tools/gather_bench 16777216 268435456 0 $b; done > gpurun_out/r4d_gather.txt 2>&1
