# end of round: smoke, full GPU suite, bench line (with the Or-opt entry), ncu full capture of the Or-opt tile sweep (C3)
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2>&1; echo bench=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:or_tile_kernel -s 2 -c 1 -o gpurun_out/oropt_tile_C3 -f python -c "
from paper_conf_ipps_rockis13_b200 import tsp2opt, inputs
c, t = inputs.config_instance('C3', 'random')
for _ in range(3): tsp2opt.oropt_best_move(c, t)
" > gpurun_out/ncu_oropt.log 2>&1; echo ncu=$?
