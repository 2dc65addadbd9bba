"""Local-search wall time with and without the CUDA-graph batches (TSP2OPT_GRAPH), per mode; results must agree."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

runs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C3:random", "C4:mf", "C5:mf", "C5:hilbert"]
for run in runs:
    cfg, start = run.split(":")
    c, t = inputs.config_instance(cfg, "random" if start == "mf" else start)
    with tsp2opt.TSP2Opt(c) as g:
        if start == "mf":
            t = g.mf_tour()["tour"]
        for mode, opt, val in (("2opt", None, 0), ("pruned8", tsp2opt.OPT_NEIGHBOURS, 8),
                               ("first", tsp2opt.OPT_FIRST_IMPROVEMENT, 1), ("2.5opt", tsp2opt.OPT_NODE_INSERTION, 1)):
            if opt is not None:
                g.set_option(opt, val)
            ref = None
            for graph in ("0", "1"):
                os.environ["TSP2OPT_GRAPH"] = graph
                g.local_search(t, max_iters=3)
                t0 = time.perf_counter()
                r = g.local_search(t)
                dt = time.perf_counter() - t0
                key = (r["iterations"], r["length"])
                ref = ref or key
                print(json.dumps({"cfg": cfg, "start": start, "mode": mode, "graph": int(graph), "iters": key[0],
                                  "length": key[1], "s": dt, "us_per_iter": 1e6 * dt / max(1, key[0]),
                                  "agrees": key == ref}), flush=True)
            if opt is not None:
                g.set_option(opt, 0)
