python tools/variants.py --configs -1 1 2 3 4 --variants default tools/alt/head.so > gpurun_out/variants.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_b.log 2>&1; echo pytest=$? >> gpurun_out/pytest_b.log
