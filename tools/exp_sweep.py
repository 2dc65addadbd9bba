"""Quick timing of the sweep kernel and local search (experiments; set TSP2OPT_LIB to pick a build).

python tools/exp_sweep.py [label]  -> one JSON line with sweep ms (C5 random/hilbert, C4 random)
and local-search wall time (C1, C2, C3 random; C4 hilbert)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

out = {"label": sys.argv[1] if len(sys.argv) > 1 else os.environ.get("TSP2OPT_LIB", "default")}
for cfg, tk in (("C5", "random"), ("C5", "hilbert"), ("C4", "random"), ("C3", "random")):
    c, t = inputs.config_instance(cfg, tk)
    with tsp2opt.TSP2Opt(c) as g:
        g.best_move(t)
        g.profile(True)
        for _ in range(5):
            mv = g.best_move()
        ms, k = g.profile_read()
        n = len(t)
        out[f"{cfg}_{tk}_sweep_ms"] = ms / k
        out[f"{cfg}_{tk}_Gpairs"] = n * (n - 1) / 2 / (ms / k) / 1e6
        out[f"{cfg}_{tk}_move"] = mv
        out["geometry_" + cfg] = g.geometry()
for cfg, tk in (("C1", "random"), ("C2", "random"), ("C3", "random"), ("C4", "hilbert")):
    c, t = inputs.config_instance(cfg, tk)
    with tsp2opt.TSP2Opt(c) as g:
        g.local_search(t, max_iters=3)
        t0 = time.perf_counter()
        r = g.local_search(t)
        out[f"LS_{cfg}_{tk}_s"] = time.perf_counter() - t0
        out[f"LS_{cfg}_{tk}_iters"] = r["iterations"]
        out[f"LS_{cfg}_{tk}_len"] = r["length"]
print(json.dumps(out))
