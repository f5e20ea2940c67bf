#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gs_ or partitioned or nccl or block_size" > gpurun_out/r2j_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2j_tests.log
timeout 900 python tools/gs_report.py --out gpurun_out/r2j_gs.jsonl > gpurun_out/r2j_gs.log 2>&1
timeout 600 python tools/dist_timing.py --configs 4 3 2 1 --out gpurun_out/r2j_dist.jsonl > gpurun_out/r2j_dist.log 2>&1
