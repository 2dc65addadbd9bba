# one gpurun call: smoke, GPU tests, bench, ncu launch list + one full capture of the sweep
set -x
mkdir -p gpurun_out
nproc; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests -m gpu -q --durations=15 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2>&1; echo bench=$?
if [ -n "$NCU" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-ls --no-cpu > gpurun_out/bench_ncu.log 2>&1; echo ncu1=$?
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/sweep_C5_random -f python tools/profile_sweep.py C5 random 2 > gpurun_out/ncu_full.log 2>&1; echo ncu2=$?
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/sweep_C5_hilbert -f python tools/profile_sweep.py C5 hilbert 2 > gpurun_out/ncu_full_h.log 2>&1; echo ncu3=$?
fi
tail -5 gpurun_out/pytest_gpu.log; tail -3 gpurun_out/bench.log
