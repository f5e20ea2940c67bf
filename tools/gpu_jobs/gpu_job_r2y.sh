#!/bin/bash
cd $GRAFT_REPO_ROOT
for c in 4 3 2; do timeout 300 python tools/round_profile_persistent.py --config $c --every 20 > gpurun_out/r2y_rounds_c$c.log 2>&1; done
