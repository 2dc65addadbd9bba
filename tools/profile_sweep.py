"""Short driver for ncu: a few sweeps of one config (python tools/profile_sweep.py C5 random 3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
tk = sys.argv[2] if len(sys.argv) > 2 else "random"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
pre = int(sys.argv[4]) if len(sys.argv) > 4 else 0  # local-search moves applied before the profiled sweeps
coords, tour = inputs.config_instance(cfg, tk)
with tsp2opt.TSP2Opt(coords) as g:
    if pre:
        tour = g.local_search(tour, max_iters=pre)["tour"]
    for _ in range(reps):
        print(g.best_move(tour), g.geometry(), flush=True)
