mkdir -p gpurun_out
TSP2OPT_TILE_BOUNDS=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/sweep_C5_random -f python tools/profile_sweep.py C5 random 2 > gpurun_out/ncu_full.log 2>&1; echo ncu2=$?
TSP2OPT_TILE_BOUNDS=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/sweep_C5_hilbert -f python tools/profile_sweep.py C5 hilbert 2 > gpurun_out/ncu_full_h.log 2>&1; echo ncu3=$?
