mkdir -p gpurun_out
# C3 mid local search (5000 moves applied): the sweep launches of 2 best_move calls; profile the 2nd
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/sweep_C3_mid -f python tools/profile_sweep.py C3 random 2 5000 > gpurun_out/ncu_c3.log 2>&1; echo c3=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/sweep_C5_random -f python tools/profile_sweep.py C5 random 2 > gpurun_out/ncu_c5.log 2>&1; echo c5=$?
