mkdir -p gpurun_out
timeout 900 python tools/exp_inc_tiling.py C4,C5 7x16,7x32,7x64,7x128 > gpurun_out/exp_inc_tiling2.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_inc_tiling2.jsonl
