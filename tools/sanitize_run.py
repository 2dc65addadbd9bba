"""One small workload per library mode, checked against the oracle, for
compute-sanitizer (memcheck / racecheck / synccheck / initcheck) runs:

    env $(python tools/sanitize_run.py --env MODE) \
        compute-sanitizer --tool memcheck python tools/sanitize_run.py MODE

Modes cover every kernel family: the persistent grid-barrier local search, the
per-iteration kernels, the culled and incremental sweeps, the cooperative
2.5-opt apply, first improvement, the pruned sweep, MF, ILS, the batched
local search and ILS, and Or-opt.  Each mode exits non-zero on a parity
mismatch; the sanitizer's own summary reports memory / race / sync errors.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

MODES = ["persistent", "kernels", "culled", "incremental", "inc3", "inc_fused", "dense_ls", "graph_off", "25opt",
         "25opt_culled", "first", "first_inc", "pruned", "mf", "ils", "batch", "batch_ils", "oropt", "oropt_filter",
         "shards", "p2p1"]

# environment each mode needs (read by the library at handle creation)
ENV = {
    "persistent": {"TSP2OPT_PERSISTENT": "1"},
    "kernels": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "1"},
    "culled": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "2", "TSP2OPT_CULL_TJ": "16"},
    "incremental": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "3", "TSP2OPT_CULL_TJ": "16"},
    "inc3": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "3", "TSP2OPT_CULL_TJ": "16",
             "TSP2OPT_INC_BARRIERS": "3"},
    "inc_fused": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "3", "TSP2OPT_CULL_TJ": "16",
                  "TSP2OPT_INC_PERSISTENT": "0"},
    "dense_ls": {"TSP2OPT_PERSISTENT": "3", "TSP2OPT_TILE_BOUNDS": "1"},
    "first_inc": {"TSP2OPT_TILE_BOUNDS": "3", "TSP2OPT_CULL_TJ": "16"},
    "graph_off": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "3", "TSP2OPT_GRAPH": "0",
                  "TSP2OPT_INC_PERSISTENT": "0"},
    "25opt_culled": {"TSP2OPT_PERSISTENT": "0", "TSP2OPT_TILE_BOUNDS": "3", "TSP2OPT_CULL_TJ": "16"},
    "oropt_filter": {"TSP2OPT_OROPT_FILTER": "1"},
}


def check(cond, what):
    if not cond:
        print("PARITY MISMATCH:", what, flush=True)
        sys.exit(3)


def main(mode):
    n = 300
    c = inputs.lattice_coords(n, 3)
    t = inputs.random_tour(n, 3)
    if mode in ("persistent", "kernels", "culled", "incremental", "inc3", "inc_fused", "dense_ls", "graph_off"):
        with tsp2opt.TSP2Opt(c) as g:
            r = g.local_search(t)
        o = oracle.local_search(c, t)
        check((r["length"], r["iterations"]) == (o["length"], o["iterations"]) and np.array_equal(r["tour"], o["tour"]),
              mode)
    elif mode in ("25opt", "25opt_culled"):
        with tsp2opt.TSP2Opt(c) as g:
            g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
            r = g.local_search(t)
        o = oracle.local_search25(c, t)
        check(r["length"] == o["length"] and np.array_equal(r["tour"], o["tour"]), mode)
    elif mode in ("first", "first_inc"):
        with tsp2opt.TSP2Opt(c) as g:
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
            r = g.local_search(t)
        o = oracle.first_local_search(c, t)
        check(r["length"] == o["length"] and np.array_equal(r["tour"], o["tour"]), mode)
    elif mode == "pruned":
        with tsp2opt.TSP2Opt(c) as g:
            g.set_option(tsp2opt.OPT_NEIGHBOURS, 8)
            r = g.local_search(t)
        o = oracle.pruned_local_search(c, t, 8)
        check(r["length"] == o["length"] and np.array_equal(r["tour"], o["tour"]), mode)
    elif mode == "mf":
        with tsp2opt.TSP2Opt(c) as g:
            m = g.mf_tour()
        check(np.array_equal(m["tour"], oracle.mf_tour(c)), mode)
    elif mode == "ils":
        with tsp2opt.TSP2Opt(c[:120]) as g:
            r = g.ils(inputs.random_tour(120, 4), 5, 11)
        o = oracle.ils(c[:120], inputs.random_tour(120, 4), 5, 11)
        check(r["length"] == o["length"], mode)
    elif mode == "batch":
        cs = np.stack([inputs.uniform_coords(100, s) for s in range(1, 9)])
        ts = np.stack([inputs.random_tour(100, s) for s in range(1, 9)])
        r = tsp2opt.batch_local_search(cs, ts)
        for b in range(8):
            check(r["lengths"][b] == oracle.local_search(cs[b], ts[b])["length"], f"batch {b}")
    elif mode == "batch_ils":
        cs = np.stack([inputs.uniform_coords(60, s) for s in range(1, 5)])
        ts = np.stack([inputs.random_tour(60, s) for s in range(1, 5)])
        seeds = np.arange(7, 11, dtype=np.uint64)
        r = tsp2opt.batch_ils(cs, ts, 4, seeds, history=False)
        for b in range(4):
            check(r["lengths"][b] == oracle.ils(cs[b], ts[b], 4, int(seeds[b]))["length"], f"batch_ils {b}")
    elif mode in ("oropt", "oropt_filter"):
        r = tsp2opt.oropt_local_search(c, t)
        o = oracle.local_search_or(c, t)
        check(r["length"] == o["length"] and np.array_equal(r["tour"], o["tour"]), mode)
    elif mode == "p2p1":  # the peer-memory exchange kernel, one rank
        with tsp2opt.TSP2Opt(c, 0, 1, p2p_allgather=lambda b: [b]) as g:
            r = g.local_search(t)
        o = oracle.local_search(c, t)
        check(r["length"] == o["length"] and np.array_equal(r["tour"], o["tour"]), mode)
    elif mode == "shards":
        with tsp2opt.TSP2Opt(c) as g:
            want = oracle.best_move(c, t)
            got = []
            for r_ in range(3):
                g.debug_set_shard(r_, 3)
                got.append(g.best_move(t))
            g.debug_set_shard(0, 1)
        best = min(got, key=lambda m: (m[2], m[1] * (m[1] - 1) // 2 + m[0]))
        check(best == want, mode)
    else:
        raise SystemExit(f"unknown mode {mode}; one of {MODES}")
    print("ok", mode, flush=True)


if __name__ == "__main__":
    if sys.argv[1] == "--env":  # the environment of a mode, for `env $(... --env MODE) compute-sanitizer ...`
        print(" ".join(f"{k}={v}" for k, v in ENV.get(sys.argv[2], {}).items()) or "TSP2OPT_NONE=1")
    elif sys.argv[1] == "--modes":
        print(" ".join(MODES))
    else:
        main(sys.argv[1])
