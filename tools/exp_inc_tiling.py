"""Incremental culled sweep: local search from MF per cull tiling (TSP2OPT_CULL_ROWS / TSP2OPT_CULL_TJ, read at
create), with the library's per-sweep event time (box + cull + list sweep).  One JSON line per run."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C4", "C5"]
variants = [v.split("x") for v in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["7x32", "7x64", "7x128", "15x32", "15x64"])]
for cfg in cfgs:
    c, _ = inputs.config_instance(cfg, "random")
    with tsp2opt.TSP2Opt(c) as g0:
        t = g0.mf_tour()["tour"]
    for rows, tj in variants:
        os.environ["TSP2OPT_CULL_ROWS"] = rows
        os.environ["TSP2OPT_CULL_TJ"] = tj
        with tsp2opt.TSP2Opt(c) as g:
            g.set_option(tsp2opt.OPT_TILE_BOUNDS, 3)
            g.local_search(t, max_iters=3)
            t0 = time.perf_counter()
            r = g.local_search(t)
            dt = time.perf_counter() - t0
            ms, launches = 0.0, 1
            if os.environ.get("EXP_PROFILE"):
                g.profile(True)
                g.local_search(t)
                ms, launches = g.profile_read()
                g.profile(False)
        print(json.dumps({"cfg": cfg, "rows": int(rows), "tj": int(tj), "iters": r["iterations"], "length": r["length"],
                          "s": dt, "us_per_iter": 1e6 * dt / max(1, r["iterations"]),
                          "sweep_us": 1e3 * ms / max(1, launches)}), flush=True)
