# GPU test run (optionally filtered: PYTEST_K='expr')
mkdir -p gpurun_out
if [ -n "$PYTEST_K" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x -k "$PYTEST_K" --durations=8 > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
else
  timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
fi
tail -12 gpurun_out/pytest_gpu.log
