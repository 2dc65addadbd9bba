"""Debug driver: the seeded mixed-operations sequence of test_seeded_sweeps_mixed_operations,
reporting the first operation after which the device state disagrees with the oracle."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

n = 3001
c = inputs.make_coords("lattice", n, 8)
t = inputs.make_tour("random", c, 8)
rng = np.random.default_rng(3)
with tsp2opt.TSP2Opt(c) as g:
    g.set_tour(t)

    def check(what):
        tour, L = g.get_tour()
        ok_perm = sorted(tour.tolist()) == list(range(n))
        Lr = oracle.tour_length(c, tour) if ok_perm else None
        bm = g.best_move()
        ref = oracle.best_move(c, tour) if ok_perm else None
        s = g.sync()
        print(what, "perm", ok_perm, "L", L, Lr, "bm", bm, ref, "it", s["iterations"], flush=True)
        if not (ok_perm and L == Lr and bm == ref):
            print("MISMATCH after", what)
            sys.exit(1)

    for rnd in range(6):
        k = int(rng.integers(1, 5))
        g.iterate_async(k)
        g.sync()
        check(f"r{rnd} iterate {k}")
        g.iterate_async(2)
        g.sync()
        check(f"r{rnd} iterate 2 after best_move")
        i, j = sorted(rng.choice(n, 2, replace=False).tolist())
        g.apply(i, j)
        g.iterate_async(1)
        g.sync()
        check(f"r{rnd} apply {i},{j} + iterate 1")
        if rnd == 3:
            g.debug_set_shard(1, 3)
            g.debug_set_shard(0, 1)
            g.iterate_async(2)
            g.sync()
            check(f"r{rnd} shard change")
        if rnd == 4:
            g.set_tour(inputs.random_tour(n, 99))
            g.iterate_async(3)
            g.sync()
            check(f"r{rnd} new tour")
print("all ok")
