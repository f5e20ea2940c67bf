#!/bin/bash
# early exit: per-round entries read (trace builds) + A/B incl. single-chunk-only exits
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python tools/variants.py --configs 1 4 8 --variants default tools/alt/noearly.so tools/alt/nomc.so > gpurun_out/r4c_variants.txt 2>&1
for v in te tne tnomc; do SGR_LIBPATH=tools/alt/$v.so timeout 300 python tools/round_profile_persistent.py --config 4 --every 10 > gpurun_out/r4c_rounds_$v.txt 2>&1; done
