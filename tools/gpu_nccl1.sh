mkdir -p gpurun_out
NCCL_DEBUG=WARN timeout 900 python -m pytest tests/test_gpu_nccl1.py -q -x --durations=5 > gpurun_out/pytest_nccl1.log 2>&1; echo pytest=$?
tail -12 gpurun_out/pytest_nccl1.log
