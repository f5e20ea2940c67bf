#!/bin/bash
# flat build: thread-per-vertex bin 0 as its own instantiation; parity + A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs or random_small or generator_families or degree_bins or overflow or block_size or loop_modes or partitioned_equals or profile_mode" > gpurun_out/r4l_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4l_tests.log
timeout 900 python tools/variants.py --configs 1 2 3 4 6 --variants default tools/alt/nofb0t.so > gpurun_out/r4l_variants.txt 2>&1
