"""C3 local search (random / MF start) per dense geometry (TSP2OPT_ROWS / TSP2OPT_TJ, read at create)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

for start in ("random", "mf"):
    c, t0 = inputs.config_instance("C3", "random")
    for rows, tj in ((7, 8), (7, 16), (7, 32), (7, 64), (15, 16), (15, 32)):
        os.environ["TSP2OPT_ROWS"] = str(rows)
        os.environ["TSP2OPT_WARPS"] = "1"
        os.environ["TSP2OPT_TJ"] = str(tj)
        with tsp2opt.TSP2Opt(c) as g:
            t = g.mf_tour()["tour"] if start == "mf" else t0
            g.local_search(t, max_iters=3)
            t1 = time.perf_counter()
            r = g.local_search(t)
            dt = time.perf_counter() - t1
        print(json.dumps({"start": start, "rows": rows, "tj": tj, "iters": r["iterations"], "length": r["length"],
                          "s": dt, "us_per_iter": 1e6 * dt / max(1, r["iterations"])}), flush=True)
