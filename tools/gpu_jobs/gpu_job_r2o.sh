#!/bin/bash
cd $GRAFT_REPO_ROOT
( time timeout 2000 python -m pytest tests -m gpu -x -q --durations=6 ) > gpurun_out/r2o_tests.log 2>&1
timeout 600 python tools/dist_timing.py --configs 2 4 3 1 --out gpurun_out/r2o_dist.jsonl > gpurun_out/r2o_dist.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2o_bench.json 2> gpurun_out/r2o_bench.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2o_smoke.log 2>&1
