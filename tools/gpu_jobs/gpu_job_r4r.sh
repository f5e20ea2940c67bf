#!/bin/bash
# T0 trimming parity + A/B; bench cfg2 reproduction (r4q bench showed 14.6 ms vs 8.5 in variants)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "flat_thread or full_size_configs or generator_families or random_small or block_size or loop_modes or profile_mode" > gpurun_out/r4r_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4r_tests.log
timeout 900 python tools/variants.py --configs 2 3 6 --variants default tools/alt/notrim.so > gpurun_out/r4r_variants.txt 2>&1
timeout 600 python bench.py --config 2 --no-cpu-baseline > gpurun_out/r4r_bench_c2.json 2> gpurun_out/r4r_bench_c2.err
python tools/dbg_c2.py > gpurun_out/r4r_dbg_c2.txt 2>&1
