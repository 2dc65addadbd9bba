"""Debug the one-barrier search: capped local searches vs the oracle, one subprocess per cap."""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 1 and sys.argv[1] == "run":
    import numpy as np
    import oracle
    from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt
    cap, n = int(sys.argv[2]), int(sys.argv[3])
    c = inputs.make_coords("lattice", n, 5)
    t = inputs.make_tour("hilbert", c, 3)
    want = oracle.local_search(c, t, max_iters=cap, trace_cap=5000)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, 5000)
        r = g.local_search(t, max_iters=cap)
        got = np.asarray(g.get_trace(5000), dtype=np.int64)
    w = want["trace"][: len(got)]
    bad = np.nonzero((got != w).any(axis=1))[0] if len(got) == len(w) else [0]
    print("cap", cap, "n", n, "it", r["iterations"], want["iterations"], "len", r["length"], want["length"],
          "first bad", bad[:1], got[bad[:1]] if len(bad) else "", w[bad[:1]] if len(bad) else "", flush=True)
else:
    env = dict(os.environ, TSP2OPT_INC_BARRIERS="1", TSP2OPT_TILE_BOUNDS="3")
    for n in (1500, 4000):
        for cap in (0, 1, 2, 5, 50, 100000):
            try:
                out = subprocess.run([sys.executable, __file__, "run", str(cap), str(n)], env=env, capture_output=True,
                                     text=True, timeout=40)
                print(out.stdout.strip() or out.stderr.strip()[-400:], flush=True)
            except subprocess.TimeoutExpired:
                print("cap", cap, "n", n, "TIMEOUT", flush=True)
