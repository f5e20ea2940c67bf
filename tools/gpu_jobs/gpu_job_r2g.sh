#!/bin/bash
# round 2: full suite + bench + Fig. 8 sweep + ldg ablation + sub-step report + sanitizers
cd $GRAFT_REPO_ROOT
( time timeout 2400 python -m pytest tests -m gpu -x -q --durations=12 ) > gpurun_out/r2g_tests.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2g_bench.json 2> gpurun_out/r2g_bench.err
timeout 900 python tools/block_sweep.py --configs 4 1 3 7 --out gpurun_out/r2g_block_sweep.jsonl > gpurun_out/r2g_block_sweep.log 2>&1
timeout 900 python tools/ldg_ablation.py --configs 4 1 3 2 7 --out gpurun_out/r2g_ldg.jsonl > gpurun_out/r2g_ldg.log 2>&1
timeout 900 python tools/gs_report.py --out gpurun_out/r2g_gs.jsonl > gpurun_out/r2g_gs.log 2>&1
for t in memcheck initcheck synccheck racecheck; do
  extra=""; [ $t = memcheck ] && extra="--leak-check full"
  timeout 1200 compute-sanitizer --tool $t $extra --print-limit 50 python tools/sanitize_run.py > gpurun_out/r2g_san_$t.log 2>&1
  echo "rc=$?" >> gpurun_out/r2g_san_$t.log
done
