mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_pruned.py -q -x > gpurun_out/pytest_pruned.log 2>&1; echo pytest_pruned=$?
tail -3 gpurun_out/pytest_pruned.log
timeout 600 python tools/exp_pruned.py C3,C4,C5 2,4 8,16 0,1 > gpurun_out/exp_pruned.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_pruned.jsonl


