# local-search breakdown for each library variant in $LIBS (path or "default"); optional tests
mkdir -p gpurun_out
for L in ${LIBS:-default}; do
  if [ "$L" = default ]; then unset TSP2OPT_LIB; else export TSP2OPT_LIB=$PWD/paper_conf_ipps_rockis13_b200/$L; fi
  python tools/exp_ls_breakdown.py ${CASES:-C3:random C4:mf C5:mf C5:hilbert} | sed "s/^{/{\"lib\": \"$L\", /" >> gpurun_out/ls_libs.jsonl 2>&1
done
unset TSP2OPT_LIB
cat gpurun_out/ls_libs.jsonl
if [ -n "$PYTEST_K" ]; then
timeout 1200 python -m pytest tests -m gpu -q -x -k "${PYTEST_K}" > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
fi
