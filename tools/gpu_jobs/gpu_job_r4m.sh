#!/bin/bash
# bin 0 groups: byte gathers + shl masks (SGR_SMALL_U8) parity + A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs or random_small or generator_families or degree_bins or overflow or block_size or loop_modes or partitioned_equals or multi_chunk or complete_graphs or self_loops" > gpurun_out/r4m_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4m_tests.log
timeout 900 python tools/variants.py --configs 1 2 3 4 6 7 --variants default tools/alt/nosu8.so > gpurun_out/r4m_variants.txt 2>&1
