#!/bin/bash
# bin-2 early exit: parity on hub graphs + A/B against the SGR_EARLY=0 build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "early_exit or multi_chunk or cfg1 or full_size_configs or random_small or generator_families or degree_bins or overflow or complete_graphs or partitioned_equals" > gpurun_out/r4b_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4b_tests.log
timeout 900 python tools/variants.py --configs 1 4 6 7 8 --variants default tools/alt/noearly.so > gpurun_out/r4b_variants.txt 2>&1
timeout 300 python tools/round_profile_persistent.py --config 4 --every 20 > gpurun_out/r4b_rounds_c4.txt 2>&1
timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r4b_bench.json 2> gpurun_out/r4b_bench.err
