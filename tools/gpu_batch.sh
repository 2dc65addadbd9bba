# batched LS: parity tests + timing sweep over block sizes and layouts
mkdir -p gpurun_out
PYTEST_K=batch bash tools/gpu_tests.sh
for PK in ${BATCH_PK:-auto}; do
for T in ${BATCH_TS:-auto 64 128 256}; do
  if [ "$T" = auto ]; then unset TSP2OPT_BATCH_THREADS; else export TSP2OPT_BATCH_THREADS=$T; fi
  if [ "$PK" = auto ]; then unset TSP2OPT_BATCH_PACKED; else export TSP2OPT_BATCH_PACKED=$PK; fi
  timeout 600 python tools/exp_batch.py
done; done > gpurun_out/exp_batch.jsonl 2>&1
cat gpurun_out/exp_batch.jsonl
