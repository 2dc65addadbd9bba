TSP2OPT_INC_TJ=64 timeout 400 python tools/exp_inc_parts.py ls1_tj64 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
TSP2OPT_INC_TJ=64 TSP2OPT_INC_PART=8 timeout 400 python tools/exp_inc_parts.py ls1_tj64_p8 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
TSP2OPT_INC_TJ=16 timeout 400 python tools/exp_inc_parts.py ls1_tj16 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
