#!/bin/bash
# T0 trimming with register compaction: parity + A/B vs old T0 (80 regs, no trim) and trim at 80 regs
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "flat_thread or full_size_configs_bit_exact and 3" > gpurun_out/r4s_tests.log 2>&1; echo pytest=$? >> gpurun_out/r4s_tests.log
timeout 900 python tools/variants.py --configs 3 6 --variants default tools/alt/t0old.so tools/alt/notrim.so tools/alt/trim768.so > gpurun_out/r4s_variants.txt 2>&1
for i in 1 2 3; do timeout 600 python bench.py --config 2 --no-cpu-baseline --no-e2e --no-secondary --steps 5 > gpurun_out/r4s_bench_c2_$i.json 2>/dev/null; done
