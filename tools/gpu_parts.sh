TSP2OPT_CULL_TJ=64 timeout 900 python tools/exp_inc_parts.py ls2_tj64 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
TSP2OPT_CULL_TJ=32 TSP2OPT_INC_PART=8 timeout 900 python tools/exp_inc_parts.py ls2_tj32_p8 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
TSP2OPT_CULL_TJ=64 TSP2OPT_INC_PART=8 timeout 900 python tools/exp_inc_parts.py ls2_tj64_p8 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
TSP2OPT_CULL_TJ=32 TSP2OPT_INC_PART=2 timeout 900 python tools/exp_inc_parts.py ls2_tj32_p2 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
TSP2OPT_CULL_TJ=32 TSP2OPT_TILE_BOUNDS=3 timeout 600 python tools/exp_c3.py c3_tb3_tj32 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
TSP2OPT_CULL_TJ=16 timeout 600 python tools/exp_c3.py c3_auto_tj16 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
TSP2OPT_CULL_TJ=32 timeout 600 python tools/exp_c3.py c3_auto_tj32 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
