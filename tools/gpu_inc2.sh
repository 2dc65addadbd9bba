mkdir -p gpurun_out
timeout 900 python tools/exp_incremental.py C4:mf,C5:mf,C5:hilbert 3 > gpurun_out/exp_inc.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_inc.jsonl
timeout 600 python tools/exp_25opt.py C4,C5 > gpurun_out/exp_25.jsonl 2>&1; cat gpurun_out/exp_25.jsonl
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --launch-skip 16000 --launch-count 2000 --csv --log-file gpurun_out/launches_inc_mid.csv python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_mid.log 2>&1; echo ncu=$?
python tools/launch_summary.py gpurun_out/launches_inc_mid.csv > gpurun_out/launches_inc_mid.txt; head -8 gpurun_out/launches_inc_mid.txt
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_25opt.py tests/test_gpu_first.py -q -x -k "incremental or seeded or culled or mixed or geometries" > gpurun_out/pytest_inc.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_inc.log
