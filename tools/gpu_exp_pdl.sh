# programmatic dependent launch on/off: local-search breakdown (library defaults); then GPU tests
mkdir -p gpurun_out
for PDL in 1 0; do
  TSP2OPT_PDL=$PDL python tools/exp_ls_breakdown.py C1:random C2:random C3:random C3:mf C4:mf C5:mf | sed "s/^{/{\"pdl\": $PDL, /" >> gpurun_out/ls_pdl.jsonl 2>&1
done
cat gpurun_out/ls_pdl.jsonl
if [ -n "$PYTEST_K" ]; then
timeout 1200 python -m pytest tests -m gpu -q -x -k "${PYTEST_K}" > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
fi
