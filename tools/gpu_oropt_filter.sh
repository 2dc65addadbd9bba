# Or-opt FP32 filter: parity in both modes, smoke, timings filtered vs unfiltered, launch times, ncu full of the filtered sweep
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 600 python -m pytest tests/test_gpu_oropt.py -x -q > gpurun_out/pytest_oropt.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_oropt.log
TSP2OPT_OROPT_FILTER=1 timeout 600 python -m pytest tests/test_gpu_oropt.py -x -q -k "best_move or local_search_parity" > gpurun_out/pytest_oropt_forcefilter.log 2>&1; echo pytest_forcefilter=$?; tail -2 gpurun_out/pytest_oropt_forcefilter.log
for F in "" 0; do
TSP2OPT_OROPT_FILTER=$F timeout 600 python -c "
import json, bench
from paper_conf_ipps_rockis13_b200 import tsp2opt
print(json.dumps(bench.time_oropt(tsp2opt, 'C1,C2,C3:hilbert,C3,C4:hilbert', False)))
" > gpurun_out/oropt_bench_filter$F.json 2>&1; echo bench$F=$?
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:or_tile_kernel -c 8 python -c "
from paper_conf_ipps_rockis13_b200 import tsp2opt, inputs
for cfg in ('C2', 'C3', 'C4', 'C5'):
    c, t = inputs.config_instance(cfg, 'random')
    tsp2opt.oropt_best_move(c, t); tsp2opt.oropt_best_move(c, t)
" > gpurun_out/ncu_oropt_times_filter.log 2>&1; echo ncu1=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:or_tile_kernel -s 2 -c 1 -o gpurun_out/oropt_tile_filter_C3h -f python -c "
from paper_conf_ipps_rockis13_b200 import tsp2opt, inputs
c, t = inputs.config_instance('C3', 'hilbert')
for _ in range(3): tsp2opt.oropt_best_move(c, t)
" > gpurun_out/ncu_oropt_filter.log 2>&1; echo ncu2=$?
