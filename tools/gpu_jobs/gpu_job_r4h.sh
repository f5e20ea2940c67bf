#!/bin/bash
# bin-2 cross-chunk pipeline: parity (default J=4) + A/B over J and off
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "early_exit or multi_chunk or cfg1 or full_size_configs or random_small or generator_families or degree_bins or complete_graphs or overflow" > gpurun_out/r4h_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4h_tests.log
timeout 900 python tools/variants.py --configs 1 4 8 --variants default tools/alt/xp2.so tools/alt/xp8.so tools/alt/noxp.so > gpurun_out/r4h_variants.txt 2>&1
