mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_batch.py -q -x -k "error or errors or invalid or explicit or sizes or device or batch_parity" > gpurun_out/pytest_e2e.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_e2e.log
timeout 600 python bench.py --steps 20 --warmup 3 --no-ls --no-cpu > gpurun_out/bench_e2e.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench_e2e.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e'])"
