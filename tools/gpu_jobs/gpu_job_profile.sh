# Per-bin cycle split, per-round times and one ncu --set full capture of the cfg4 round kernel
python tools/bin_cycles.py 2 3 4 > gpurun_out/bin_cycles.txt 2>&1
python tools/round_profile_persistent.py --config 4 --every 20 > gpurun_out/round_c4.txt 2>&1
python tools/round_profile_persistent.py --config 2 --every 40 > gpurun_out/round_c2.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persistent -c 1 \
  -o gpurun_out/full_c4 -f python tools/run_once.py --config 4 --loop-mode persistent > gpurun_out/ncu_full_c4.log 2>&1
echo done
