#!/bin/bash
cd $GRAFT_REPO_ROOT
python tools/variants.py --configs 2 3 --variants default tools/alt/nodense.so tools/alt/cap768.so tools/alt/cap1280.so tools/alt/cap1056nd.so > gpurun_out/r2f_variants.txt 2>&1
python tools/round_profile_persistent.py --config 2 --every 20 > gpurun_out/r2f_round_c2.txt 2>&1
SGR_LIBPATH=tools/alt/nodense.so python tools/round_profile_persistent.py --config 2 --every 20 > gpurun_out/r2f_round_c2_nodense.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gs_" > gpurun_out/r2f_gs_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2f_gs_tests.log
