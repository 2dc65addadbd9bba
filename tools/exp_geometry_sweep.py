"""Single-sweep device time vs geometry (R, warps, TJ) for one config (sweep-kernel CUDA events)."""
import itertools
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
name, _, tk = cfg.partition(":")
c, t = inputs.config_instance(name, tk or None)
for R, W, TJ in itertools.product((7, 15), (1, 2, 4), (32, 64, 128, 256, 512, 1024)):
    os.environ.update(TSP2OPT_ROWS=str(R), TSP2OPT_WARPS=str(W), TSP2OPT_TJ=str(TJ))
    with tsp2opt.TSP2Opt(c) as g:
        geo = g.geometry()
        if geo["tiles"] < 300:
            continue
        g.best_move(t)
        g.profile(True)
        for _ in range(3):
            g.best_move()
        ms, k = g.profile_read()
        print(json.dumps(dict(cfg=cfg, R=R, W=W, TJ=TJ, tiles=geo["tiles"], sweep_ms=round(ms / k, 4))), flush=True)
