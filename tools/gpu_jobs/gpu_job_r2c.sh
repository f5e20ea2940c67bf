#!/bin/bash
# round 2: A/B of async bin-2 gathers + bench.py line check
cd $GRAFT_REPO_ROOT
python tools/variants.py --configs 4 1 --variants default tools/alt/a512.so tools/alt/a1024.so tools/alt/a256.so > gpurun_out/r2c_variants.txt 2>&1
timeout 900 python bench.py --config 4 --steps 10 --warmup 3 > gpurun_out/r2c_bench.json 2> gpurun_out/r2c_bench.err
