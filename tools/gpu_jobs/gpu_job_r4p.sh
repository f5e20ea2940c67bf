#!/bin/bash
# dense passes: double-buffered stage; parity + A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs or generator_families or block_size or random_small" > gpurun_out/r4p_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4p_tests.log
timeout 900 python tools/variants.py --configs 2 --variants default tools/alt/nodb.so > gpurun_out/r4p_variants.txt 2>&1
