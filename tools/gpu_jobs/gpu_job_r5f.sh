#!/bin/bash
# final build: smoke + bench lines of the configs the size-dependent bins changed, and the headline
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r5f_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r5f_smoke.log
timeout 600 python bench.py > gpurun_out/r5f_bench.json 2> gpurun_out/r5f_bench.err
for c in 1 6 7; do timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/r5f_bench_c$c.json 2>> gpurun_out/r5f_bench.err; done
