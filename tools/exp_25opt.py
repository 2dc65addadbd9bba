"""2.5-opt experiment: local search from MF (and one dense random-tour sweep) per config.
One JSON line per run: iterations, length, seconds, us per iteration, sweep us (library events)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C3", "C4", "C5"]
for cfg in cfgs:
    c, tr = inputs.config_instance(cfg, "random")
    n = len(c)
    with tsp2opt.TSP2Opt(c) as g:
        t = g.mf_tour()["tour"]
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
        g.local_search(t, max_iters=3)
        g.profile(True)
        t0 = time.perf_counter()
        r = g.local_search(t)
        dt = time.perf_counter() - t0
        ms, launches = g.profile_read()
        g.profile(False)
        # one dense sweep of a random tour (no tile bound skips: every pair is checked)
        g.profile(True)
        for _ in range(3):
            g.best_move(tr)
        ms2, l2 = g.profile_read()
        g.profile(False)
        print(json.dumps({"cfg": cfg, "n": n, "iters": r["iterations"], "length": r["length"], "s": dt,
                          "us_per_iter": 1e6 * dt / max(1, r["iterations"]), "sweep_us": 1e3 * ms / max(1, launches),
                          "random_sweep_ms": ms2 / max(1, l2),
                          "random_pairs_per_s": n * (n - 1) / 2 / (ms2 / max(1, l2) * 1e-3)}), flush=True)
