#!/bin/bash
cd $GRAFT_REPO_ROOT
python tools/variants.py --configs 4 3 2 --variants default > gpurun_out/r2i_variants.txt 2>&1
SGR_L2PERSIST=1 python tools/variants.py --configs 4 3 2 --variants tools/alt/../../paper_conf_ipps_licqfsty16_b200/lib/libsgr.so >> gpurun_out/r2i_variants.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gs_" > gpurun_out/r2i_gs_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2i_gs_tests.log
timeout 900 python tools/gs_report.py --out gpurun_out/r2i_gs.jsonl > gpurun_out/r2i_gs.log 2>&1
timeout 600 python tools/dist_timing.py --configs 4 3 2 1 --out gpurun_out/r2i_dist.jsonl > gpurun_out/r2i_dist.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2i_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-secondary > gpurun_out/r2i_ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persistent -c 1 -o gpurun_out/r2i_full_c4 -f python tools/run_once.py --config 4 --loop-mode persistent > gpurun_out/r2i_ncu_full.log 2>&1
