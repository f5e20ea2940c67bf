#!/bin/bash
# ncu --set full of the dense-pass kernel on cfg2 (27-point stencil 104^3)
cd $GRAFT_REPO_ROOT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_dense -c 1 \
  -o gpurun_out/r2z_dense_c2 -f python tools/run_once.py --config 2 --loop-mode persistent > gpurun_out/r2z_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_persistent -s 1 -c 1 \
  -o gpurun_out/r2z_flat_c2 -f python tools/run_once.py --config 2 --loop-mode persistent >> gpurun_out/r2z_ncu.log 2>&1
echo done >> gpurun_out/r2z_ncu.log
