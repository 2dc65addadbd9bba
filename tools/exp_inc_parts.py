"""Persistent incremental local search: kept tiles swept whole by one warp (TSP2OPT_INC_PART=0) or split
into column parts over the CTA's warps; time per move and the result vs the committed golden file.
    TSP2OPT_INC_PART=K python tools/exp_inc_parts.py LABEL"""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

GOLD = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden")
label = sys.argv[1] if len(sys.argv) > 1 else "default"
runs = [("C4", "hilbert", "radius"), ("C4", "mf", "radius"), ("C5", "hilbert", "radius"), ("C5", "mf", "radius"),
        ("C4", "mf", "first"), ("C5", "mf", "first")]
out = {"label": label, "env": {k: v for k, v in os.environ.items() if k.startswith("TSP2OPT_")}}
for cfg, tk, var in runs:
    coords, tour = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    gold = np.load(os.path.join(GOLD, f"ls_{var}_{cfg}_lattice_{tk}_s1.npz"))
    best = None
    with tsp2opt.TSP2Opt(coords) as g:
        if var == "first":
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
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
    k = f"{cfg}_{tk}_{var}"
    out[k + "_s"] = round(best, 4)
    out[k + "_us_per_move"] = round(best / max(1, r["iterations"]) * 1e6, 2)
    out[k + "_golden_equal"] = bool(ok)
    print(k, out[k + "_s"], out[k + "_us_per_move"], ok, flush=True, file=sys.stderr)
print(json.dumps(out), flush=True)
