"""Phase clocks of the persistent incremental local search (build with
`python -m paper_conf_ipps_rockis13_b200._build --variant phase -DTSP2OPT_PHASE_TIMING`,
run with TSP2OPT_LIB=<that .so>): cycles per move of each phase, CTA 0."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

names = ["boxes", "barrier1", "cull+sweep", "barrier2", "apply", "barrier3", "clean_scan", "-",
         "max_warp_cull+sweep", "max_warp_sweeps", "max_warp_first_cull", "kept_tiles(count)"]
for cfg, tk in (("C4", "hilbert"), ("C5", "hilbert"), ("C5", "mf")):
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        if tk == "mf":
            g.mf_tour()
        tsp2opt.debug_phases(True)
        r = g.local_search_current() if tk == "mf" else g.local_search(t)
        ph = tsp2opt.debug_phases(True)
    k = max(1, r["iterations"])
    print(json.dumps({"config": cfg, "start": tk, "moves": r["iterations"],
                      "us_per_move_at_1.9GHz": {nm: round(v / k / (1.0 if "count" in nm else 1900.0), 3)
                                                for nm, v in zip(names, ph) if nm != "-"}}),
          flush=True)
