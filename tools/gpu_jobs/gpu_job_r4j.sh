#!/bin/bash
# dense passes: byte gathers + bit masks (SGR_DENSE_U8) parity + A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs or random_small or generator_families or degree_bins or overflow or complete_graphs or block_size" > gpurun_out/r4j_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4j_tests.log
timeout 900 python tools/variants.py --configs 2 3 --variants default tools/alt/nou8.so > gpurun_out/r4j_variants.txt 2>&1
