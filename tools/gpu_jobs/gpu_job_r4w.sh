#!/bin/bash
# flat_bin0 hook tests + compute-sanitizer over every kernel family (incl. this session's paths)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "flat_bin0 or flat_thread or dense or random_small" > gpurun_out/r4w_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4w_tests.log
for t in memcheck initcheck synccheck racecheck; do
  extra=""; [ $t = memcheck ] && extra="--leak-check full"
  timeout 900 compute-sanitizer --tool $t $extra python tools/sanitize_run.py > gpurun_out/r4w_san_$t.log 2>&1; echo rc=$? >> gpurun_out/r4w_san_$t.log
done
for c in 2 3; do timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/r4w_bench_c$c.json 2>> gpurun_out/r4w_bench.err; done
