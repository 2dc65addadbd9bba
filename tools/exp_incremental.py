"""Local search wall time per TSP2OPT_OPT_TILE_BOUNDS (1 in-sweep bound, 2 culled, 3 culled + incremental)
per config and start; results must agree across modes.  One JSON line per run."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

runs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C3:random", "C3:mf", "C4:mf", "C4:hilbert", "C5:mf", "C5:hilbert"]
modes = [int(x) for x in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["1", "2", "3"])]
for run in runs:
    cfg, start = run.split(":")
    c, t = inputs.config_instance(cfg, "random" if start == "mf" else start)
    with tsp2opt.TSP2Opt(c) as g:
        if start == "mf":
            t = g.mf_tour()["tour"]
        ref = None
        for m in modes:
            g.set_option(tsp2opt.OPT_TILE_BOUNDS, m)
            g.local_search(t, max_iters=3)
            t0 = time.perf_counter()
            r = g.local_search(t)
            dt = time.perf_counter() - t0
            key = (r["iterations"], r["length"])
            ref = ref or key
            print(json.dumps({"cfg": cfg, "start": start, "tile_bounds": m, "iters": r["iterations"],
                              "length": r["length"], "s": dt, "us_per_iter": 1e6 * dt / max(1, r["iterations"]),
                              "agrees": key == ref}), flush=True)
