bash tools/gpu.sh exp:default,base,r112,r104,lb20 > /dev/null 2>&1
timeout 600 python tools/exp_c3.py default 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
TSP2OPT_TILE_BOUNDS=3 timeout 600 python tools/exp_c3.py tb3 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
TSP2OPT_TILE_BOUNDS=3 TSP2OPT_CULL_TJ=16 timeout 600 python tools/exp_c3.py tb3_tj16 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
timeout 900 python tools/exp_c3_switch.py 2>&1 | tee gpurun_out/exp_c3_switch.jsonl
