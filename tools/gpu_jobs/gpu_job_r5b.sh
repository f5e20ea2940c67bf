#!/bin/bash
# degree-bin boundary sweep on the current kernels (cfg4, cfg1, cfg8)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for c in 4 1 8; do timeout 600 python tools/bins_sweep.py $c; done > gpurun_out/r5b_bins.txt 2>&1
