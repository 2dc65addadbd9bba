"""First vs best improvement: local search wall time, moves, length per config/start (library defaults)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

runs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C1:random", "C2:random", "C3:random", "C3:mf", "C4:mf", "C5:mf"]
for run in runs:
    cfg, start = run.split(":")
    c, t = inputs.config_instance(cfg, "random" if start == "mf" else start)
    with tsp2opt.TSP2Opt(c) as g:
        if start == "mf":
            t = g.mf_tour()["tour"]
        for first in (0, 1):
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, first)
            g.local_search(t, max_iters=3)
            t0 = time.perf_counter()
            r = g.local_search(t)
            dt = time.perf_counter() - t0
            print(json.dumps({"cfg": cfg, "start": start, "first": first, "iters": r["iterations"],
                              "length": r["length"], "s": dt, "us_per_iter": 1e6 * dt / max(1, r["iterations"])}),
                  flush=True)
