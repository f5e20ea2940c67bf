#!/bin/bash
# size-dependent default med_max: parity + timing vs the previous default
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 700 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "cfg1 or random_small or generator_families or multi_chunk or early_exit or complete_graphs or overflow or block_size or host_batch or partitioned_equals or flat_bin0 or bin0_colors" > gpurun_out/r5d_tests.log 2>&1; echo pytest=$? >> gpurun_out/r5d_tests.log
timeout 500 python tools/variants.py --configs 1 6 7 4 --variants default tools/alt/pf2.so > gpurun_out/r5d_variants.txt 2>&1
