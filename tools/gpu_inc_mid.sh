mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --launch-skip 16000 --launch-count 2000 --csv --log-file gpurun_out/launches_inc_mid.csv python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_mid.log 2>&1; echo ncu=$?
python tools/launch_summary.py gpurun_out/launches_inc_mid.csv > gpurun_out/launches_inc_mid.txt; head -10 gpurun_out/launches_inc_mid.txt
