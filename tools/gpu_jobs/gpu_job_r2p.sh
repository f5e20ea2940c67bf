#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 1200 python tools/occupancy_ab.py default:256 tools/alt/mt576.so:192 tools/alt/mt640.so:160 tools/alt/mt768.so:128 tools/alt/mt768.so:160 tools/alt/mt576.so:256 default:192 > gpurun_out/r2p_occ.txt 2>&1
