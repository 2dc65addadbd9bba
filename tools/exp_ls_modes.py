"""Local-search wall time, persistent single launch vs per-iteration kernels."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

for mode in ("1", "0"):
    os.environ["TSP2OPT_PERSISTENT"] = mode
    out = {"persistent": mode}
    for cfg, tk in (("C1", "random"), ("C2", "random"), ("C3", "random"), ("C4", "hilbert")):
        c, t = inputs.config_instance(cfg, tk)
        with tsp2opt.TSP2Opt(c) as g:
            g.local_search(t, max_iters=3)
            t0 = time.perf_counter()
            r = g.local_search(t)
            out[f"{cfg}_{tk}"] = [round(time.perf_counter() - t0, 4), r["iterations"]]
    print(json.dumps(out), flush=True)
