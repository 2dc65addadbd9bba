timeout 900 python tools/exp_inc_parts.py ls2_default 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
for K in 1 2; do TSP2OPT_INC_DIAG_PART=$K timeout 900 python tools/exp_inc_parts.py ls2_diag$K 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl; done
TSP2OPT_INC_PART=8 TSP2OPT_INC_DIAG_PART=2 timeout 900 python tools/exp_inc_parts.py ls2_p8_diag2 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
