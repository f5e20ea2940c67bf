#!/bin/bash
cd $GRAFT_REPO_ROOT
for c in 1 2 3 6 7 8 5; do timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e; done > gpurun_out/r2l_bench_other.jsonl 2> gpurun_out/r2l_bench_other.err
python tools/round_profile_persistent.py --config 4 --every 10 > gpurun_out/r2l_round_c4.txt 2>&1
