"""How much of each local-search sweep the tile bound skips (instrumented build, TSP2OPT_LIB=
libtsp2opt_stats.so): tiles walked / tiles swept, warp column steps, exact-path steps."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

CASES = [tuple(a.split(":")) for a in sys.argv[1:]] or [("C3", "random"), ("C4", "mf"), ("C5", "mf")]
for cfg, tk in CASES:
    c, t = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
    with tsp2opt.TSP2Opt(c) as g:
        geo = g.geometry()
        if tk == "mf":
            t = g.mf_tour()["tour"]
        tsp2opt.debug_stats(True)
        t0 = time.perf_counter()
        r = g.local_search(t)
        dt = time.perf_counter() - t0
        st = tsp2opt.debug_stats(True)
        sweeps = r["iterations"] + 1
        st.update(cfg=cfg, start=tk, geo=geo, walked_per_sweep=round(st["tiles_walked"] / (r["iterations"] + 1)), s=round(dt, 4), iters=r["iterations"],
                  walked_frac=round(st["tiles_walked"] / (sweeps * geo["tiles"] * geo["warps"]), 5),
                  steps_per_sweep=round(st["warp_steps"] / sweeps), pairs_per_sweep=geo["pairs"])
        print(json.dumps(st), flush=True)
