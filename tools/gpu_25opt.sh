mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_25opt.py -q -x --durations=8 > gpurun_out/pytest_25.log 2>&1; echo pytest_25=$?
tail -25 gpurun_out/pytest_25.log
timeout 600 python tools/exp_25opt.py C3,C4,C5 > gpurun_out/exp_25opt.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_25opt.jsonl
