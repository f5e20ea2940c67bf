#!/bin/bash
# GS variants: huge members one block each; parity (O3) + report vs the warp-only build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gs_" > gpurun_out/r5k_tests.log 2>&1; echo pytest=$? >> gpurun_out/r5k_tests.log
timeout 700 python tools/gs_report.py --configs 3 4 --reps 2 --out gpurun_out/r5k_gs.jsonl > gpurun_out/r5k_gs.log 2>&1
SGR_LIBPATH=tools/alt/gsold.so timeout 700 python tools/gs_report.py --configs 4 --reps 2 --out gpurun_out/r5k_gs_old.jsonl > gpurun_out/r5k_gs_old.log 2>&1
