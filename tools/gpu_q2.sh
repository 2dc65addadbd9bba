mkdir -p gpurun_out
timeout 600 python tools/exp_incremental.py C4:mf,C4:hilbert,C5:mf,C5:hilbert 3 > gpurun_out/exp_inc.jsonl 2>&1; cat gpurun_out/exp_inc.jsonl
timeout 600 python tools/exp_25opt.py C4,C5 > gpurun_out/exp_25.jsonl 2>&1; cat gpurun_out/exp_25.jsonl
timeout 600 python tools/exp_first.py C4:mf,C5:mf > gpurun_out/exp_first.jsonl 2>&1; cat gpurun_out/exp_first.jsonl
