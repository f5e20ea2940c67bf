#!/bin/bash
# round 2: dense flat passes: parity subset + A/B timing
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -x -q -k "not cfg5 and not nnz_beyond" > gpurun_out/r2d_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2d_tests.log
python tools/variants.py --configs 2 3 1 4 --variants default tools/alt/nodense.so tools/alt/div4.so tools/alt/div8.so > gpurun_out/r2d_variants.txt 2>&1
