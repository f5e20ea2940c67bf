#!/bin/bash
# HEAD check after session restore: smoke, full GPU suite, headline bench, launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r4a_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r4a_smoke.log
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=25 ) > gpurun_out/r4a_pytest.log 2>&1; echo pytest=$? >> gpurun_out/r4a_pytest.log
timeout 600 python bench.py > gpurun_out/r4a_bench.json 2> gpurun_out/r4a_bench.err
for c in 2 3; do timeout 600 python bench.py --config $c --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/r4a_bench_c$c.json 2>> gpurun_out/r4a_bench.err; done
