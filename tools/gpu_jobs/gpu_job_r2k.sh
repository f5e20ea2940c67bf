#!/bin/bash
cd $GRAFT_REPO_ROOT
python tools/variants.py --configs 2 3 1 4 7 --variants default tools/alt/nostage.so > gpurun_out/r2k_variants.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "generator_families or random_small or full_size_configs or block_size or degree_bins or loop_modes or partitioned" > gpurun_out/r2k_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2k_tests.log
