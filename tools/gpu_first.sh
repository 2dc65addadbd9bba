mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_first.py -q -x --durations=8 > gpurun_out/pytest_first.log 2>&1; echo pytest_first=$?
tail -14 gpurun_out/pytest_first.log
timeout 900 python tools/exp_first.py > gpurun_out/exp_first.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_first.jsonl
