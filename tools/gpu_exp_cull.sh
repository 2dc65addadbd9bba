# culled-sweep tiling: local-search breakdown vs TSP2OPT_CULL_ROWS x TSP2OPT_CULL_TJ; then the GPU tests
mkdir -p gpurun_out
for R in ${CULL_ROWS:-15}; do for TJ in ${CULL_TJS:-16 32 64 128}; do
  TSP2OPT_TILE_BOUNDS=2 TSP2OPT_CULL_ROWS=$R TSP2OPT_CULL_TJ=$TJ python tools/exp_ls_breakdown.py ${CASES:-C3:random C3:mf C4:mf C5:mf} | sed "s/^{/{\"cull_rows\": $R, \"cull_tj\": $TJ, /" >> gpurun_out/ls_cull_tj.jsonl 2>&1
done; done
cat gpurun_out/ls_cull_tj.jsonl
if [ -n "$PYTEST_K" ]; then
timeout 1200 python -m pytest tests -m gpu -q -x -k "${PYTEST_K}" > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
fi
