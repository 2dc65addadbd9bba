mkdir -p gpurun_out
timeout 900 python tools/exp_gseed.py > gpurun_out/exp_gseed.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_gseed.jsonl
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "local_search or seeded or shards or trace or max_iters" > gpurun_out/pytest_gs.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_gs.log
