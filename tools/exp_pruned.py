"""Pruned-sweep experiment: local search from MF per TSP2OPT_PRUNED_TP, per config and K.
Prints one JSON line per run (pruned sweep avg us from the library's events, us per iteration)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C3", "C4", "C5"]
tps = [int(x) for x in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["1", "2", "4", "8"])]
bycity = [int(x) for x in (sys.argv[4].split(",") if len(sys.argv) > 4 else ["1"])]
Ks = [int(x) for x in (sys.argv[3].split(",") if len(sys.argv) > 3 else ["8", "16"])]
for cfg in cfgs:
    c, _ = inputs.config_instance(cfg)
    with tsp2opt.TSP2Opt(c) as g:
        t = g.mf_tour()["tour"]
        for K in Ks:
            g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
            for tp, bc in [(a, b) for a in tps for b in bycity]:
                os.environ["TSP2OPT_PRUNED_TP"] = str(tp)
                os.environ["TSP2OPT_PRUNED_BYCITY"] = str(bc)
                g.local_search(t, max_iters=3)
                g.profile(True)
                t0 = time.perf_counter()
                r = g.local_search(t)
                dt = time.perf_counter() - t0
                ms, launches = g.profile_read()
                g.profile(False)
                print(json.dumps({"cfg": cfg, "K": K, "tp": tp, "bycity": bc, "iters": r["iterations"], "length": r["length"],
                                  "s": dt, "us_per_iter": 1e6 * dt / max(1, r["iterations"]),
                                  "sweep_us": 1e3 * ms / max(1, launches)}), flush=True)
