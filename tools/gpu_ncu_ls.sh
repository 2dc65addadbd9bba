# C5 local search from the MF start, 4000 moves in: launch list of 3 iterations + full ncu of one culled sweep
mkdir -p gpurun_out
timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5_mf_ls.csv python tools/profile_sweep.py C5 mf 3 4000 > gpurun_out/ncu_l.log 2>&1; echo launches=$?
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:sweep_list -s 1 -c 1 -o gpurun_out/sweep_C5_mf_ls -f python tools/profile_sweep.py C5 mf 2 4000 > gpurun_out/ncu_c5.log 2>&1; echo full=$?
