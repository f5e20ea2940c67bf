# parity suite + A/B timing of the default build (and any variants passed as args)
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$? | tee -a gpurun_out/pytest_gpu.log
python tools/variants.py --configs 2 3 4 --variants default "$@" > gpurun_out/variants.txt 2>&1
python tools/bin_cycles.py 4 > gpurun_out/bin_cycles.txt 2>&1
