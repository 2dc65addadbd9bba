"""C3 random-start local search: from the state after k dense-loop moves, time the rest of the search with
the dense loop (in-sweep tile bound, TILE_BOUNDS 1) and with the persistent incremental search (3)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

coords, tour = inputs.config_instance("C3", "random")
with tsp2opt.TSP2Opt(coords) as g:
    for k in (0, 1000, 2000, 4000, 6000, 8000, 9000):
        g.set_option(tsp2opt.OPT_TILE_BOUNDS, 1)
        r0 = g.local_search(tour, max_iters=k) if k else {"tour": tour, "iterations": 0}
        t_k = r0["tour"]
        res = {"k": k}
        for tb in (1, 3):
            g.set_option(tsp2opt.OPT_TILE_BOUNDS, tb)
            best = None
            for rep in range(2):
                t0 = time.perf_counter()
                r = g.local_search(t_k)
                dt = time.perf_counter() - t0
                best = dt if best is None else min(best, dt)
            res[f"tb{tb}_s"] = round(best, 4)
            res[f"tb{tb}_moves"] = r["iterations"]
            res[f"tb{tb}_us_per_move"] = round(best / max(1, r["iterations"]) * 1e6, 2)
            res[f"tb{tb}_length"] = r["length"]
        print(json.dumps(res), flush=True)
