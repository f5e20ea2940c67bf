#!/bin/bash
# round 2: full -m gpu suite (incl. cfg5) + bench lines for cfg4/3/2
cd $GRAFT_REPO_ROOT
nproc > gpurun_out/r2a_nproc.txt; lscpu | grep "Model name" >> gpurun_out/r2a_nproc.txt
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 ) > gpurun_out/r2a_tests.log 2>&1
for c in 4 3 2; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e; done > gpurun_out/r2a_bench.jsonl 2> gpurun_out/r2a_bench.err
