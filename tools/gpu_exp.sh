# experiment call: tests (quick subset or full), then exp_sweep for each lib variant given in $LIBS
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
for L in $LIBS; do
  TSP2OPT_LIB=$L timeout 600 python tools/exp_sweep.py $L >> gpurun_out/exp.jsonl 2>gpurun_out/exp_err.log; echo exp=$?
done
cat gpurun_out/exp.jsonl
