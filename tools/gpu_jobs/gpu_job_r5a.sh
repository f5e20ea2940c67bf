#!/bin/bash
# end-of-session check: smoke, full GPU suite, cfg2 bench (dense stage-ahead build)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r5a_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r5a_smoke.log
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=5 ) > gpurun_out/r5a_pytest.log 2>&1; echo pytest=$? >> gpurun_out/r5a_pytest.log
for i in 1 2; do timeout 600 python bench.py --config 2 --no-cpu-baseline > gpurun_out/r5a_bench_c2_$i.json 2>> gpurun_out/r5a_bench.err; done
