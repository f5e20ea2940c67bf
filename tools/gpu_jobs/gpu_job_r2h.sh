#!/bin/bash
# round 2: parity suite (dist device path, small masks, TMA fix) + sanitizers + A/B + bench + sweeps
cd $GRAFT_REPO_ROOT
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=8 -k "not nnz_beyond and not cfg5_full" ) > gpurun_out/r2h_tests.log 2>&1
for t in memcheck initcheck synccheck racecheck; do
  extra=""; [ $t = memcheck ] && extra="--leak-check full"
  timeout 900 compute-sanitizer --tool $t $extra --print-limit 30 python tools/sanitize_run.py > gpurun_out/r2h_san_$t.log 2>&1
  echo "rc=$?" >> gpurun_out/r2h_san_$t.log
done
python tools/variants.py --configs 4 3 2 1 7 --variants default tools/alt/nosmall.so > gpurun_out/r2h_variants.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2h_bench.json 2> gpurun_out/r2h_bench.err
timeout 600 python tools/dist_timing.py --configs 4 3 2 1 --out gpurun_out/r2h_dist.jsonl > gpurun_out/r2h_dist.log 2>&1
timeout 900 python tools/block_sweep.py --configs 4 1 3 7 --reps 3 --out gpurun_out/r2h_block_sweep.jsonl > gpurun_out/r2h_block_sweep.log 2>&1
