mkdir -p gpurun_out
timeout 900 python tools/exp_graph.py > gpurun_out/exp_graph.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_graph.jsonl
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pruned.py tests/test_gpu_first.py tests/test_gpu_25opt.py -q -x -k "local_search or mixed or incremental or trace" > gpurun_out/pytest_graph.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_graph.log
