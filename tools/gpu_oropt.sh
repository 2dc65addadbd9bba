# Or-opt: GPU parity tests, smoke, the Or-opt bench entries, ncu of the Or-opt sweep
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
tail -2 gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_oropt.py -x -q --durations=8 > gpurun_out/pytest_oropt.log 2>&1; echo pytest=$?
tail -15 gpurun_out/pytest_oropt.log
TSP2OPT_OROPT_NAIVE=1 timeout 900 python -m pytest tests/test_gpu_oropt.py -x -q -k "best_move or local_search_parity" > gpurun_out/pytest_oropt_naive.log 2>&1; echo pytest_naive=$?
tail -2 gpurun_out/pytest_oropt_naive.log
TSP2OPT_OROPT_NAIVE=1 timeout 600 python -c "
import json, bench
from paper_conf_ipps_rockis13_b200 import tsp2opt
print(json.dumps(bench.time_oropt(tsp2opt, 'C2,C3:hilbert', False)))
" > gpurun_out/oropt_bench_naive.json 2>&1; echo bench_naive=$?
timeout 600 python -c "
import json, bench
from paper_conf_ipps_rockis13_b200 import tsp2opt
print(json.dumps(bench.time_oropt(tsp2opt, 'C1,C2,C3:hilbert,C3', True)))
" > gpurun_out/oropt_bench.json 2> gpurun_out/oropt_bench.err; echo bench=$?
cat gpurun_out/oropt_bench.json | head -c 3000
timeout 600 ncu --set full --clock-control none -k regex:or_tile_kernel -s 3 -c 1 -o gpurun_out/oropt_sweep -f python -c "
from paper_conf_ipps_rockis13_b200 import tsp2opt, inputs
c, t = inputs.config_instance('C3', 'random')
for _ in range(5): tsp2opt.oropt_best_move(c, t)
" > gpurun_out/ncu_oropt.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_oropt.log
