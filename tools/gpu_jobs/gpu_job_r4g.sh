#!/bin/bash
# claim atomics without immediate consumers: parity subset + A/B vs the previous default
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "early_exit or multi_chunk or cfg1 or full_size_configs or random_small or generator_families or degree_bins or partitioned_equals or dense" > gpurun_out/r4g_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4g_tests.log
timeout 900 python tools/variants.py --configs 1 2 3 4 8 --variants default tools/alt/noearly.so > gpurun_out/r4g_variants.txt 2>&1
