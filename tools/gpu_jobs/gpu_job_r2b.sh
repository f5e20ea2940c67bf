#!/bin/bash
# round 2: per-round times (persistent) + ncu --set full of fat host-mode passes (cfg4)
cd $GRAFT_REPO_ROOT
python tools/round_profile_persistent.py --config 4 --every 10 > gpurun_out/r2b_round_c4.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 12 \
  -o gpurun_out/r2b_host_c4 -f python tools/run_once.py --config 4 --loop-mode host > gpurun_out/r2b_ncu.log 2>&1
echo done
