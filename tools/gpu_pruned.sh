# pruned-neighbourhood round: its GPU tests, the quick full suite, the bench line
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_pruned.py -q -x --durations=10 > gpurun_out/pytest_pruned.log 2>&1; echo pytest_pruned=$?
tail -15 gpurun_out/pytest_pruned.log
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps(d.get('pruned_local_search'), indent=0)); print(d['value'])"
