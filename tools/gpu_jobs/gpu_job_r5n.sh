#!/bin/bash
# GS in-place mode with block-per-huge-vertex: properness tests + report
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gs_" > gpurun_out/r5n_tests.log 2>&1; echo pytest=$? >> gpurun_out/r5n_tests.log
timeout 700 python tools/gs_report.py --configs 3 4 --reps 2 --out gpurun_out/r5n_gs.jsonl > gpurun_out/r5n_gs.log 2>&1
