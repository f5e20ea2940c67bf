#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "generator_families or random_small or full_size_configs or block_size or degree_bins or loop_modes or edge_cases or self_loops or overflow" > gpurun_out/r2r_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2r_tests.log
python tools/variants.py --configs 2 3 1 4 --variants default tools/alt/nodense.so tools/alt/div4.so > gpurun_out/r2r_variants.txt 2>&1
python tools/round_profile_persistent.py --config 2 --every 20 > gpurun_out/r2r_round_c2.txt 2>&1
