"""Short driver for ncu: a few sweeps of one config (python tools/profile_sweep.py C5 random 3 [pre]).
tk = random | hilbert | mf.  `pre` local-search moves are applied first (not profiled: the
sweeps are bracketed by cudaProfilerStart/Stop, use ncu --profile-from-start off)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
tk = sys.argv[2] if len(sys.argv) > 2 else "random"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
pre = int(sys.argv[4]) if len(sys.argv) > 4 else 0  # local-search moves applied before the profiled sweeps
coords, tour = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
with tsp2opt.TSP2Opt(coords) as g:
    if tk == "mf":
        tour = g.mf_tour()["tour"]
    if pre:
        tour = g.local_search(tour, max_iters=pre)["tour"]
    g.set_tour(tour)
    torch.cuda.profiler.start()
    for _ in range(reps):
        g.iterate_async(1)
        print(g.sync(), g.geometry(), flush=True)
    torch.cuda.profiler.stop()
