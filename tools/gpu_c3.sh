mkdir -p gpurun_out
for tj in 8 16; do export TSP2OPT_CULL_TJ=$tj; echo "tj=$tj"; timeout 600 python tools/exp_incremental.py C3:random,C3:mf,C3:hilbert 1,3; done > gpurun_out/exp_c3.jsonl 2>&1
cat gpurun_out/exp_c3.jsonl
