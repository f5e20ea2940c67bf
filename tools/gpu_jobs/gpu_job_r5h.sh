#!/bin/bash
# final HEAD: smoke + full GPU suite
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r5h_smoke.log 2>&1; echo smoke=$? >> gpurun_out/r5h_smoke.log
( time timeout 1500 python -m pytest tests -m gpu -x -q --durations=5 ) > gpurun_out/r5h_pytest.log 2>&1; echo pytest=$? >> gpurun_out/r5h_pytest.log
