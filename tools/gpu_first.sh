mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_first.py tests/test_gpu_pruned.py -q -x --durations=5 -k "pruned" > gpurun_out/pytest_first.log 2>&1; echo pytest_first=$?
tail -8 gpurun_out/pytest_first.log
