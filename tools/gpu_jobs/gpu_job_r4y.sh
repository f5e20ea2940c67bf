#!/bin/bash
# dense passes: offsets two words ahead (SGR_DENSE_PF2) A/B + parity of that build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 400 python tools/variants.py --configs 2 --variants default tools/alt/pf2.so > gpurun_out/r4y_variants.txt 2>&1
SGR_LIBPATH=tools/alt/pf2.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense or full_size_configs_bit_exact and 2 or generator_families or flat_bin0" > gpurun_out/r4y_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4y_tests.log
