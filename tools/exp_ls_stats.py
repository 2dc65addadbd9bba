"""Local-search totals with seeding on/off (TSP2OPT_SEED), per-iteration kernels (TSP2OPT_PERSISTENT=0)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

for seed in ("1", "0"):
    os.environ["TSP2OPT_SEED"] = seed
    for cfg, tk in (("C2", "random"), ("C3", "random"), ("C4", "hilbert")):
        c, t = inputs.config_instance(cfg, tk)
        with tsp2opt.TSP2Opt(c) as g:
            g.local_search(t, max_iters=2)
            tsp2opt.debug_stats(True)
            t0 = time.perf_counter()
            r = g.local_search(t)
            dt = time.perf_counter() - t0
            st = tsp2opt.debug_stats(True)
            st.update(seed=seed, cfg=cfg, tour=tk, s=round(dt, 4), iters=r["iterations"],
                      slow_frac=round(st["slow_steps"] / max(1, st["warp_steps"]), 4))
            print(json.dumps(st), flush=True)
