#!/bin/bash
# hub bin 1: rows staged one step ahead by TMA; parity + A/B (short timeouts: mbarrier code)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 120 python tools/run_once.py --config 1 --loop-mode persistent > gpurun_out/r4t_once.log 2>&1; echo once=$? >> gpurun_out/r4t_once.log
timeout 400 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "multi_chunk or early_exit or cfg1 or full_size_configs or random_small or generator_families or degree_bins or overflow or complete_graphs or block_size or loop_modes or partitioned_equals" > gpurun_out/r4t_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4t_tests.log
timeout 400 python tools/variants.py --configs 1 4 7 8 --variants default tools/alt/nob1s.so > gpurun_out/r4t_variants.txt 2>&1
