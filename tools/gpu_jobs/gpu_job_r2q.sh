#!/bin/bash
cd $GRAFT_REPO_ROOT
python tools/variants.py --configs 4 7 1 --variants default tools/alt/noid2.so tools/alt/noid4.so tools/alt/qb4.so > gpurun_out/r2q_variants.txt 2>&1
