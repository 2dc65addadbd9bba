mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "incremental or seeded or shards or local_search_parity" > gpurun_out/pytest_inc.log 2>&1; echo pytest_inc=$?
tail -3 gpurun_out/pytest_inc.log
timeout 900 python tools/exp_incremental.py C3:random,C3:mf,C4:mf,C4:hilbert,C5:mf,C5:hilbert 1,2,3 > gpurun_out/exp_inc.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_inc.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_inc_C5.csv python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_inc.log 2>&1; echo ncu=$?
python tools/launch_summary.py gpurun_out/launches_inc_C5.csv > gpurun_out/launches_inc_C5.txt; head -8 gpurun_out/launches_inc_C5.txt
