#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "dense_passes or generator_families or random_small or full_size_configs or loop_modes or edge_cases" > gpurun_out/r2t_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2t_tests.log
python tools/variants.py --configs 2 3 1 4 --variants default tools/alt/nodense.so tools/alt/span4.so > gpurun_out/r2t_variants.txt 2>&1
