#!/bin/bash
# dense passes: next word's offsets prefetched, threshold n/8; parity + A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs or generator_families or block_size" > gpurun_out/r4o_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4o_tests.log
timeout 900 python tools/variants.py --configs 2 --variants default tools/alt/dd8.so tools/alt/pfdd16.so > gpurun_out/r4o_variants.txt 2>&1
