"""Filter statistics of the persistent incremental search (TSP2OPT_STATS build via TSP2OPT_LIB):
column steps, steps on the rare path and exact candidates per move."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

for cfg, tk in (("C4", "hilbert"), ("C5", "hilbert"), ("C5", "mf"), ("C3", "mf")):
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        if tk == "mf":
            g.mf_tour()
        tsp2opt.debug_stats(True)
        r = g.local_search_current() if tk == "mf" else g.local_search(t)
        st = tsp2opt.debug_stats(True)
    k = max(1, r["iterations"])
    print(json.dumps({"config": cfg, "start": tk, "moves": k, "warp_steps_per_move": st["warp_steps"] / k,
                      "slow_steps_per_move": st["slow_steps"] / k, "slow_frac": st["slow_steps"] / max(1, st["warp_steps"]),
                      "exact_pairs_per_move": st["exact_pairs"] / k, "tiles_walked_per_move": st["tiles_walked"] / k}),
          flush=True)
