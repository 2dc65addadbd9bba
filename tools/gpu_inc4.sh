mkdir -p gpurun_out
for g in 0 1184 592 296; do
  export TSP2OPT_LIST_GRID=$g
  echo "list_grid=$g"
  timeout 600 python tools/exp_incremental.py C4:mf,C5:mf,C5:hilbert 3
done > gpurun_out/exp_inc4.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_inc4.jsonl
