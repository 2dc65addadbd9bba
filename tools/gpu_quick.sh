mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_25opt.py tests/test_gpu_parity.py -q -x -k "25 or incremental or seeded" > gpurun_out/pytest_q.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_q.log
timeout 600 python tools/exp_25opt.py C3,C4,C5 > gpurun_out/exp_25opt.jsonl 2>&1; echo exp25=$?
cat gpurun_out/exp_25opt.jsonl
timeout 600 python tools/exp_incremental.py C4:mf,C5:mf,C5:hilbert 3 > gpurun_out/exp_inc.jsonl 2>&1; echo expinc=$?
cat gpurun_out/exp_inc.jsonl
