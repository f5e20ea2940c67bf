#!/bin/bash
# session-3 checkpoint: smoke, full GPU suite, bench lines (headline + every config + reference arm), launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r4q_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r4q_smoke.log
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=10 ) > gpurun_out/r4q_pytest.log 2>&1; echo pytest=$? >> gpurun_out/r4q_pytest.log
timeout 600 python bench.py > gpurun_out/r4q_bench.json 2> gpurun_out/r4q_bench.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r4q_bench_ref.json 2>> gpurun_out/r4q_bench.err
for c in 1 2 3 5 6 7 8; do timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/r4q_bench_c$c.json 2>> gpurun_out/r4q_bench.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r4q_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/r4q_ncu_bench.log 2>&1
