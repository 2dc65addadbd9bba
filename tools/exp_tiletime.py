"""Per-tile clocks of the sweep (needs the TSP2OPT_TILE_TIMING build via TSP2OPT_LIB):
prologue (loads, staging, seed key) and walk cycles per walked tile, and the slowest tile."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

for cfg, tk, what in (("C5", "random", "sweep"), ("C3", "random", "ls"), ("C3", "mf", "ls"), ("C4", "hilbert", "ls"),
                      ("C5", "hilbert", "ls")):
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        if tk == "mf":
            g.mf_tour()
        tsp2opt.debug_stats(True)
        if what == "sweep":
            mv = g.best_move(t)
            k = 1
        else:
            r = g.local_search_current() if tk == "mf" else g.local_search(t)
            k = max(1, r["iterations"])
        st = tsp2opt.debug_stats(True)
    pro, walk, tiles, mx = st["warp_steps"], st["slow_steps"], st["exact_pairs"], st["tiles_walked"]
    print(json.dumps({"config": cfg, "start": tk, "what": what, "iterations": k, "tiles_per_it": tiles / k,
                      "prologue_cyc_per_tile": pro / max(1, tiles), "walk_cyc_per_tile": walk / max(1, tiles),
                      "max_tile_cyc": mx}), flush=True)
