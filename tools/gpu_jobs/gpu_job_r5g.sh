#!/bin/bash
# T0 bin 0 rows by per-lane TMA bulk copies: parity + A/B (short timeouts: mbarrier code)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 120 python tools/run_once.py --config 3 --loop-mode persistent > gpurun_out/r5g_once.log 2>&1; echo once=$? >> gpurun_out/r5g_once.log
timeout 500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "flat_bin0 or flat_thread or full_size_configs_bit_exact or random_small or bin0_colors or generator_families" > gpurun_out/r5g_tests.log 2>&1; echo pytest=$? >> gpurun_out/r5g_tests.log
timeout 400 python tools/variants.py --configs 3 2 --variants default tools/alt/notma.so > gpurun_out/r5g_variants.txt 2>&1
