#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs_bit_exact or gs_" > gpurun_out/r3b_tests.log 2>&1; echo pytest=$? >> gpurun_out/r3b_tests.log
timeout 300 python bench.py --config 2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/r3b_bench_c2.json 2> gpurun_out/r3b_bench_c2.err
timeout 300 python tools/round_profile_persistent.py --config 2 --every 40 > gpurun_out/r3b_rounds_c2.log 2>&1
timeout 600 python tools/gs_report.py --configs 3 4 --out gpurun_out/r3b_gs.jsonl > gpurun_out/r3b_gs.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_dense -c 1 \
  -o gpurun_out/r3b_dense_c2 -f python tools/run_once.py --config 2 --loop-mode persistent > gpurun_out/r3b_ncu.log 2>&1
