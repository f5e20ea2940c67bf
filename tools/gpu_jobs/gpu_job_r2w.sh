#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gs_" > gpurun_out/r2w_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2w_tests.log
timeout 900 python tools/gs_report.py --out gpurun_out/r2w_gs.jsonl > gpurun_out/r2w_gs.log 2>&1
