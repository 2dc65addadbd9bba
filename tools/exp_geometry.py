"""Local-search wall time and first-sweep time vs sweep geometry (R, warps, TJ) via env overrides."""
import itertools
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C2", "C3"]
for cfg in cfgs:
    name, _, tk = cfg.partition(":")
    c, t = inputs.config_instance(name, tk or None)
    for R, W, TJ in itertools.product((7, 15), (1, 2, 4), (8, 16, 32, 64, 128, 256)):
        os.environ.update(TSP2OPT_ROWS=str(R), TSP2OPT_WARPS=str(W), TSP2OPT_TJ=str(TJ))
        with tsp2opt.TSP2Opt(c) as g:
            geo = g.geometry()
            if geo["tiles"] < 100:
                continue
            g.local_search(t, max_iters=2)
            t0 = time.perf_counter()
            r = g.local_search(t)
            dt = time.perf_counter() - t0
            print(json.dumps(dict(cfg=cfg, R=R, W=W, TJ=TJ, tiles=geo["tiles"], ls_s=round(dt, 4),
                                  iters=r["iterations"])), flush=True)
