#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "partitioned or nccl" > gpurun_out/r2n_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2n_tests.log
timeout 600 python tools/dist_timing.py --configs 2 4 3 1 --out gpurun_out/r2n_dist.jsonl > gpurun_out/r2n_dist.log 2>&1
