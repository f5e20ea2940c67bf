#!/bin/bash
cd $GRAFT_REPO_ROOT
python tools/variants.py --configs 2 --variants default tools/alt/pipe512.so tools/alt/pipe768.so tools/alt/nopipe512.so > gpurun_out/r2v_variants.txt 2>&1
