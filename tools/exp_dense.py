"""A/B timing of library builds (experiments): `TSP2OPT_LIB=<so> python tools/exp_dense.py LABEL`.

One JSON line: the dense C5 / C4 sweep as bench.py's `value` times it (tile bounds
off, every pair tested; the library's per-launch CUDA events, warm, 10 sweeps),
with the move for a parity cross-check, and the wall time to a local minimum
for C3 random and C5 Hilbert in the library's default configuration.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

out = {"label": sys.argv[1] if len(sys.argv) > 1 else "default", "lib": os.path.basename(tsp2opt.LIB),
       "env": {k: v for k, v in os.environ.items() if k.startswith("TSP2OPT_") and k != "TSP2OPT_LIB"}}
for cfg in ("C5", "C4"):
    c, t = inputs.config_instance(cfg, "random")
    n = len(t)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_TILE_BOUNDS, 0)
        mv = g.best_move(t)
        g.profile(True)
        for _ in range(10):
            g.best_move()
        ms, k = g.profile_read()
        out[f"{cfg}_dense_ms"] = round(ms / k, 4)
        out[f"{cfg}_Tpairs"] = round(n * (n - 1) / 2 / (ms / k) / 1e9, 4)
        out[f"{cfg}_move"] = mv
for cfg, tk in (("C3", "random"), ("C4", "hilbert"), ("C5", "hilbert"), ("C5", "mf")):
    if os.environ.get("EXP_NO_LS"):
        break
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        if tk == "mf":
            g.mf_tour()
            g.local_search_current(max_iters=3)
            g.mf_tour()
            t0 = time.perf_counter()
            r = g.local_search_current()
        else:
            g.local_search(t, max_iters=3)
            t0 = time.perf_counter()
            r = g.local_search(t)
        dt = time.perf_counter() - t0
        out[f"LS_{cfg}_{tk}_s"] = round(dt, 4)
        out[f"LS_{cfg}_{tk}_us_per_move"] = round(1e6 * dt / max(1, r["iterations"]), 2)
        out[f"LS_{cfg}_{tk}"] = [r["iterations"], r["length"]]
print(json.dumps(out), flush=True)
