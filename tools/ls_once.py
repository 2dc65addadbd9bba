"""One local search through the library (for ncu launch lists / sanitizers):
    python tools/ls_once.py CFG START [MAX_ITERS] [first|25opt|knn8]
START = random | hilbert | mf.  Prints the result line."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfg, tk = sys.argv[1], sys.argv[2]
cap = int(sys.argv[3]) if len(sys.argv) > 3 and int(sys.argv[3]) >= 0 else None
variant = sys.argv[4] if len(sys.argv) > 4 else ""
coords, tour = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
with tsp2opt.TSP2Opt(coords) as g:
    if variant == "first":
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
    elif variant == "25opt":
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
    elif variant.startswith("knn"):
        g.set_option(tsp2opt.OPT_NEIGHBOURS, int(variant[3:]))
    if tk == "mf":
        g.mf_tour()
        r = g.local_search_current(max_iters=cap)
    else:
        r = g.local_search(tour, max_iters=cap)
    print({k: v for k, v in r.items() if k != "tour"}, flush=True)
