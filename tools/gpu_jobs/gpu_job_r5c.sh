#!/bin/bash
# degree-bin boundary sweep on the 2^20-vertex Table I shapes
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for c in 6 7; do timeout 600 python tools/bins_sweep.py $c; done > gpurun_out/r5c_bins.txt 2>&1
