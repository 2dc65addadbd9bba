#!/bin/bash
# compute-sanitizer over every library mode (tools/sanitize_run.py); summaries -> gpurun_out/sanitize/
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/sanitize
python -c "import oracle; oracle.build()"
for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  for m in ${MODES:-$(python tools/sanitize_run.py --modes)}; do
    env $(python tools/sanitize_run.py --env $m) timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool $tool \
      --print-limit 20 python tools/sanitize_run.py $m > gpurun_out/sanitize/${tool}_${m}.log 2>&1
    echo "$tool $m rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|^ok |MISMATCH' gpurun_out/sanitize/${tool}_${m}.log | tr '\n' ' ')"
  done
done | tee gpurun_out/sanitize/summary.txt
