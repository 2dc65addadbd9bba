"""Dense best-improvement local search with and without the global seed (TSP2OPT_GLOBAL_SEED, read at create)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

runs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C2:random", "C3:random", "C3:mf", "C4:random"]
for run in runs:
    cfg, start = run.split(":")
    c, t = inputs.config_instance(cfg, "random" if start == "mf" else start)
    ref = None
    for gs in ("0", "1"):
        os.environ["TSP2OPT_GLOBAL_SEED"] = gs
        with tsp2opt.TSP2Opt(c) as g:
            if start == "mf":
                t = g.mf_tour()["tour"]
            g.set_option(tsp2opt.OPT_PERSISTENT, 0)
            if cfg == "C4":
                g.set_option(tsp2opt.OPT_TILE_BOUNDS, 1)
            cap = 3000 if cfg == "C4" else None
            g.local_search(t, max_iters=3)
            t0 = time.perf_counter()
            r = g.local_search(t, max_iters=cap)
            dt = time.perf_counter() - t0
        key = (r["iterations"], r["length"])
        ref = ref or key
        print(json.dumps({"cfg": cfg, "start": start, "global_seed": int(gs), "iters": key[0], "length": key[1], "s": dt,
                          "us_per_iter": 1e6 * dt / max(1, key[0]), "agrees": key == ref}), flush=True)
