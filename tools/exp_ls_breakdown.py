"""Where does local-search time go?  Sum of sweep-kernel device time (CUDA events around every
sweep launch) vs the wall time of tsp2opt_local_search (library-default loop), from the
random / Hilbert / Multiple Fragment starts."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

CASES = [("C2", "random"), ("C3", "random"), ("C3", "mf"), ("C4", "hilbert"), ("C4", "mf"), ("C5", "mf")]
if len(sys.argv) > 1:
    CASES = [tuple(a.split(":")) for a in sys.argv[1:]]
for cfg, tk in CASES:
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        g.local_search(t, max_iters=2)
        if tk == "mf":
            t = g.mf_tour()["tour"]
        g.profile(True)
        t0 = time.perf_counter()
        r = g.local_search(t)
        dt = time.perf_counter() - t0
        ms, k = g.profile_read()
        g.profile(False)
        print(json.dumps(dict(cfg=cfg, start=tk, wall_s=round(dt, 4), sweep_s=round(ms / 1e3, 4), sweeps=k,
                              iters=r["iterations"], per_iter_us=round(dt / max(1, r["iterations"]) * 1e6, 2),
                              sweep_us=round(ms * 1e3 / max(1, k), 2))), flush=True)
