#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "generator_families or random_small or full_size_configs or block_size or degree_bins" > gpurun_out/r2e_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2e_tests.log
python tools/variants.py --configs 2 3 --variants default tools/alt/nodense.so tools/alt/db16.so tools/alt/db4.so tools/alt/div4.so > gpurun_out/r2e_variants.txt 2>&1
