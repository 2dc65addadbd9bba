"""Filter statistics per sweep (needs the TSP2OPT_STATS build via TSP2OPT_LIB)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

res = []
for cfg, tk, pre in (("C3", "random", 0), ("C3", "random", 2000), ("C3", "random", 8000), ("C5", "random", 0),
                     ("C5", "hilbert", 0), ("C4", "hilbert", 2000)):
    c, t = inputs.config_instance(cfg, tk)
    with tsp2opt.TSP2Opt(c) as g:
        if pre:
            r = g.local_search(t, max_iters=pre)
            t = r["tour"]
        g.best_move(t)
        tsp2opt.debug_stats(True)
        g.profile(True)
        mv = g.best_move()
        ms, _ = g.profile_read()
        st = tsp2opt.debug_stats(True)
        n = len(t)
        st.update(cfg=cfg, tour=tk, after_moves=pre, move=mv, sweep_ms=ms, pairs=n * (n - 1) // 2,
                  slow_frac=st["slow_steps"] / max(1, st["warp_steps"]),
                  exact_per_pair=st["exact_pairs"] / (n * (n - 1) / 2))
        res.append(st)
        print(json.dumps(st), flush=True)
