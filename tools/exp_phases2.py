"""Phase clocks of the two-barrier persistent incremental search (inc_ls2_kernel; build with
`python -m paper_conf_ipps_rockis13_b200._build --variant phase -DTSP2OPT_PHASE_TIMING`, run with
TSP2OPT_LIB=<that .so>): microseconds per move of CTA 0's phases and the per-move maxima over CTAs."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

names = {0: "C", 1: "barrier1", 2: "X", 3: "barrier2", 12: "max_cull", 13: "max_stage", 14: "max_items",
         15: "max_kept_per_cta(count)",
         8: "max_C", 9: "max_X"}
for cfg, tk in (("C4", "hilbert"), ("C5", "hilbert"), ("C5", "mf")):
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        if tk == "mf":
            g.mf_tour()
        tsp2opt.debug_phases(True)
        r = g.local_search_current() if tk == "mf" else g.local_search(t)
        ph = tsp2opt.debug_phases(True)
    k = max(1, ph[10])
    print(json.dumps({"config": cfg, "start": tk, "moves": r["iterations"], "counted": ph[10],
                      "us_per_move_at_1.9GHz": {nm: round(ph[q] / k / (1.0 if 'count' in nm else 1900.0), 3) for q, nm in names.items()}}),
          flush=True)
