#!/bin/bash
# round-2 final state: smoke, full GPU suite, bench lines (headline, reference arm, every config),
# launch list, ncu --set full of cfg2 / cfg3 (round kernels + k_dense) for ncu_traffic.json
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r4v_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r4v_smoke.log
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=10 ) > gpurun_out/r4v_pytest.log 2>&1; echo pytest=$? >> gpurun_out/r4v_pytest.log
timeout 600 python bench.py > gpurun_out/r4v_bench.json 2> gpurun_out/r4v_bench.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r4v_bench_ref.json 2>> gpurun_out/r4v_bench.err
for c in 1 2 3 5 6 7 8 2; do timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/r4v_bench_c$c.json 2>> gpurun_out/r4v_bench.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r4v_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/r4v_ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none -k "regex:k_persistent|k_dense" -c 4 -o gpurun_out/r4v_full_c2 -f python tools/run_once.py --config 2 --loop-mode persistent > gpurun_out/r4v_ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none -k "regex:k_persistent|k_dense" -c 4 -o gpurun_out/r4v_full_c3 -f python tools/run_once.py --config 3 --loop-mode persistent > gpurun_out/r4v_ncu_c3.log 2>&1
