#!/bin/bash
# dense passes: next word staged into the other half-stage ahead (SGR_DENSE_AHEAD) A/B + parity of that build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 400 python tools/variants.py --configs 2 --variants default tools/alt/ah.so > gpurun_out/r4x_variants.txt 2>&1
SGR_LIBPATH=tools/alt/ah.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs_bit_exact and 2 or generator_families or flat_bin0" > gpurun_out/r4x_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4x_tests.log
