#!/bin/bash
# multi-chunk bin-2 vertices decided by their last chunk (SGR_TICKET): parity + A/B
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 120 python tools/run_once.py --config 1 --loop-mode persistent > gpurun_out/r4z_once.log 2>&1; echo once=$? >> gpurun_out/r4z_once.log
timeout 700 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "multi_chunk or early_exit or cfg1 or full_size_configs or random_small or generator_families or degree_bins or overflow or complete_graphs or block_size or loop_modes or partitioned or nccl or step" > gpurun_out/r4z_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4z_tests.log
timeout 500 python tools/variants.py --configs 1 4 7 8 --variants default tools/alt/notk.so tools/alt/tk256.so tools/alt/tk16.so > gpurun_out/r4z_variants.txt 2>&1
