#!/bin/bash
# extra parity cases: flat kernels with int32 words and block sizes
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "int32_words_and_block_sizes or flat_bin0_thread_families" > gpurun_out/r5j_tests.log 2>&1; echo pytest=$? >> gpurun_out/r5j_tests.log
