"""C3 local searches (random and MF starts) under the current environment; time per move and the result
vs the committed golden files.    TSP2OPT_...=... python tools/exp_c3.py LABEL"""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

GOLD = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden")
label = sys.argv[1] if len(sys.argv) > 1 else "default"
out = {"label": label, "env": {k: v for k, v in os.environ.items() if k.startswith("TSP2OPT_")}}
for tk, gf in (("random", "ls_C3_lattice_random_s1.npz"), ("mf", "ls_radius_C3_lattice_mf_s1.npz"),
               ("hilbert", "ls_radius_C3_lattice_hilbert_s1.npz")):
    coords, tour = inputs.config_instance("C3", "random" if tk == "mf" else tk)
    gold = np.load(os.path.join(GOLD, gf))
    best = None
    with tsp2opt.TSP2Opt(coords) as g:
        for rep in range(3):
            if tk == "mf":
                g.mf_tour()
            t0 = time.perf_counter()
            r = g.local_search_current() if tk == "mf" else g.local_search(tour)
            dt = time.perf_counter() - t0
            best = dt if best is None else min(best, dt)
        ftour, _ = g.get_tour()
    ok = (r["iterations"] == int(gold["iterations"]) and r["length"] == int(gold["length"])
          and np.array_equal(ftour, gold["tour"]))
    out[f"C3_{tk}_s"] = round(best, 4)
    out[f"C3_{tk}_us_per_move"] = round(best / max(1, r["iterations"]) * 1e6, 2)
    out[f"C3_{tk}_golden_equal"] = bool(ok)
print(json.dumps(out), flush=True)
