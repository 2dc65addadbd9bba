# local-search breakdown: culled sweep (default) vs in-sweep tile bounds, + the instrumented cull stats
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -k "${PYTEST_K:-gpu}" > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
for B in ${BOUNDS:-2 1}; do
  TSP2OPT_TILE_BOUNDS=$B python tools/exp_ls_breakdown.py | sed "s/^/{\"bounds\": $B, /; s/, {/, /" >> gpurun_out/ls_breakdown.jsonl 2>&1
done
TSP2OPT_LIB=$PWD/paper_conf_ipps_rockis13_b200/libtsp2opt_stats.so python tools/exp_ls_cull.py > gpurun_out/ls_cull.jsonl 2>&1
cat gpurun_out/ls_breakdown.jsonl gpurun_out/ls_cull.jsonl
