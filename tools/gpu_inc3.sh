mkdir -p gpurun_out
for v in "" v8 box216; do
  if [ -z "$v" ]; then export TSP2OPT_LIB=; unset TSP2OPT_LIB; else export TSP2OPT_LIB=$PWD/paper_conf_ipps_rockis13_b200/libtsp2opt_$v.so; fi
  echo "variant=$v"
  timeout 600 python tools/exp_incremental.py C4:mf,C5:mf,C5:hilbert 3
done > gpurun_out/exp_inc3.jsonl 2>&1; echo exp=$?
cat gpurun_out/exp_inc3.jsonl
