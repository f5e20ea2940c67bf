python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$? >> gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$? >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2>> gpurun_out/bench.err
for c in 1 2 3 6 7 8; do timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_c$c.json 2>> gpurun_out/bench.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persistent -c 1 -o gpurun_out/full_c4 -f python tools/run_once.py --config 4 --loop-mode persistent > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_persistent -c 2 -o gpurun_out/full_c2 -f python tools/run_once.py --config 2 --loop-mode persistent > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_persistent -c 2 -o gpurun_out/full_c3 -f python tools/run_once.py --config 3 --loop-mode persistent > /dev/null 2>&1
python tools/round_profile_persistent.py --config 4 --every 20 > gpurun_out/round_c4.txt 2>&1
