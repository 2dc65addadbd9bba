mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_switches.py tests/test_gpu_ils_variants.py tests/test_gpu_pruned.py tests/test_gpu_first.py tests/test_gpu_25opt.py -q -x -k "switch or threads or ils or errors or mixed" --durations=6 > gpurun_out/pytest_misc.log 2>&1; echo pytest=$?
tail -10 gpurun_out/pytest_misc.log
