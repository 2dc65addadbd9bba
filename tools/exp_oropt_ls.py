"""Or-opt local search wall time per config (tsp2opt_oropt_local_search, host tour in and out)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt
for cfg, tk in (("C1","random"),("C2","random"),("C3","hilbert"),("C3","random")):
    c, t = inputs.config_instance(cfg, tk)
    tsp2opt.oropt_local_search(c, t, max_iters=2)
    t0 = time.perf_counter(); r = tsp2opt.oropt_local_search(c, t); dt = time.perf_counter() - t0
    print(json.dumps({"oropt": cfg, "start": tk, "s": round(dt,4), "moves": r["iterations"], "us_per_move": round(1e6*dt/max(1,r["iterations"]),1), "length": r["length"]}), flush=True)
