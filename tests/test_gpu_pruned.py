"""GPU parity of the neighbourhood-pruned 2-opt (TSP2OPT_OPT_NEIGHBOURS;
SURVEY.md §8(f) NEXT-4; L18 §V / L26 §VII; reading R18) against
oracle.pruned_* -- bit-exact: (i, j, delta) per sweep, final tour, length and
move count, through the C ABI."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu

SIZES = [3, 4, 5, 7, 16, 33, 100, 481, 1002, 2500]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_pruned_best_move_parity(gpu, n, kind):
    c = inputs.make_coords(kind, n, 5)
    with tsp2opt.TSP2Opt(c) as g:
        for K in (1, 2, 5, 8, 16):
            g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
            nb = oracle.knn(c, K)
            for t in (inputs.random_tour(n, 5), inputs.random_tour(n, 6), inputs.hilbert_tour(c)):
                assert g.best_move(t) == oracle.pruned_best_move(c, t, K, nbr=nb), K


def test_pruned_ties_duplicates_collinear(gpu):
    grid = np.array([[x * 300, y * 300] for x in range(20) for y in range(15)], dtype=np.int32)
    dup = inputs.make_coords("uniform", 200, 9)
    dup[50:60] = dup[7]  # ten copies of one city: d = 0 and id ties in the lists
    line = np.array([[(97 * k) % 30000, 12345] for k in range(150)], dtype=np.int32)
    for c in (grid, dup, line):
        n = len(c)
        with tsp2opt.TSP2Opt(c) as g:
            for K in (3, 8, 16):
                g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
                t = inputs.random_tour(n, K)
                assert g.best_move(t) == oracle.pruned_best_move(c, t, K)
                res = g.local_search(t)
                want = oracle.pruned_local_search(c, t, K)
                assert (res["length"], res["iterations"]) == (want["length"], want["iterations"])
                assert np.array_equal(res["tour"], want["tour"])


@pytest.mark.parametrize("kind,n,seed", [("uniform", 100, 1), ("uniform", 1002, 2), ("lattice", 1002, 1),
                                         ("uniform", 3000, 3), ("lattice", 7397, 1)])
@pytest.mark.parametrize("K", [4, 8, 16])
def test_pruned_local_search_trace(gpu, kind, n, seed, K):
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    cap = 10 * n
    want = oracle.pruned_local_search(c, t, K, trace_cap=cap)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
        g.set_option(tsp2opt.OPT_TRACE, cap)
        res = g.local_search(t)
        trace = g.get_trace(cap)
    assert res["status"] == want["status"] == tsp2opt.OK
    assert res["iterations"] == want["iterations"] and res["length"] == want["length"]
    assert np.array_equal(res["tour"], want["tour"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), want["trace"])


def test_pruned_max_iters(gpu):
    c = inputs.make_coords("uniform", 1002, 4)
    t = inputs.random_tour(1002, 4)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_NEIGHBOURS, 6)
        for cap in (0, 1, 7, 100):
            res = g.local_search(t, max_iters=cap)
            want = oracle.pruned_local_search(c, t, 6, max_iters=cap)
            assert res["status"] == want["status"] == tsp2opt.MAXITER
            assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
            assert np.array_equal(res["tour"], want["tour"])


def test_pruned_mixed_operations(gpu):
    """The inverse permutation the enumeration needs must follow every state
    change: explicit apply, a new tour, switching the neighbourhood off and on,
    the device-side loop, and a shard change."""
    n, K = 1500, 8
    c = inputs.make_coords("lattice", n, 2)
    t = inputs.random_tour(n, 2)
    nb = oracle.knn(c, K)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_tour(t)  # tour loaded before the option: pos is built when K is set
        g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
        cur = t.copy()
        assert g.best_move() == oracle.pruned_best_move(c, cur, K, nbr=nb)
        for i, j in ((0, 1), (3, 900), (0, n - 1), (n - 2, n - 1), (17, 18), (200, 1400)):
            g.apply(i, j)
            cur = oracle.apply(cur, i, j)
            assert g.best_move() == oracle.pruned_best_move(c, cur, K, nbr=nb)
        g.set_option(tsp2opt.OPT_NEIGHBOURS, 0)  # full neighbourhood on the same tour
        assert g.best_move() == oracle.best_move(c, cur)
        m0 = g.sync()["iterations"]
        g.iterate_async(5)  # full-neighbourhood moves while pos is not maintained
        assert g.sync()["iterations"] == m0 + 5
        for _ in range(5):
            i, j, d = oracle.best_move(c, cur)
            cur = oracle.apply(cur, i, j)
        g.set_option(tsp2opt.OPT_NEIGHBOURS, K)  # pos rebuilt from the current tour
        g.iterate_async(7)  # no best_move first: the pending key must not leak across neighbourhoods
        g.sync()
        for _ in range(7):
            i, j, d = oracle.pruned_best_move(c, cur, K, nbr=nb)
            cur = oracle.apply(cur, i, j)
        assert np.array_equal(g.get_tour()[0], cur)
        assert g.best_move() == oracle.pruned_best_move(c, cur, K, nbr=nb)
        t2 = inputs.random_tour(n, 77)
        assert g.best_move(t2) == oracle.pruned_best_move(c, t2, K, nbr=nb)  # a new tour rebuilds pos
        # simulated shards: positions split in `world` ranges, min over shards
        want = oracle.pruned_best_move(c, t2, K, nbr=nb)
        for world in (2, 3, 8):
            keys = []
            for r in range(world):
                g.debug_set_shard(r, world)
                i, j, d = g.best_move()
                keys.append((d, j * (j - 1) // 2 + i, i, j))
            d, _, i, j = min(keys)
            assert (i, j, d) == want, world
        g.debug_set_shard(0, 1)


def test_pruned_option_errors(gpu):
    c = inputs.make_coords("uniform", 50, 1)
    with tsp2opt.TSP2Opt(c) as g:
        for bad in (-1, tsp2opt.MAX_NEIGHBOURS + 1):
            with pytest.raises(tsp2opt.TSP2OptError):
                g.set_option(tsp2opt.OPT_NEIGHBOURS, bad)
        g.set_option(tsp2opt.OPT_NEIGHBOURS, 4)
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 0)  # switching a mode off is always valid
        with pytest.raises(tsp2opt.TSP2OptError):
            g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)  # exclusive with pruning


@pytest.mark.parametrize("cfg", ["C4", "C5"])
def test_pruned_full_size_from_mf(gpu, cfg):
    """At BASELINE.json sizes from the Multiple Fragment start (K = 8): the
    traced moves replayed on the CPU give the final tour and length; sampled
    iterations re-swept by the oracle (list enumeration) give the traced move;
    the pruned minimum carries the oracle's pruned certificate; the full
    neighbourhood continued from it ends at a full 2-opt local minimum."""
    K = 8
    c, t0 = inputs.config_instance(cfg, "random")
    n = len(c)
    cap = 4 * n
    nb = oracle.knn(c, K)
    with tsp2opt.TSP2Opt(c) as g:
        t = g.mf_tour()["tour"]
        g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
        g.set_option(tsp2opt.OPT_TRACE, cap)
        res = g.local_search(t)
        trace = g.get_trace(cap)
        g.set_option(tsp2opt.OPT_NEIGHBOURS, 0)
        g.set_option(tsp2opt.OPT_TRACE, 0)
        full = g.local_search_current()
        full["tour"] = g.get_tour()[0]
    k = res["iterations"]
    assert res["status"] == tsp2opt.OK and len(trace) == k > 0
    picks = set(np.linspace(0, k - 1, 6).astype(int).tolist())
    tour = t.copy()
    L = oracle.tour_length(c, tour)
    for idx, (i, j, d) in enumerate(trace):
        if idx in picks:
            assert oracle.pruned_best_move(c, tour, K, nbr=nb) == (int(i), int(j), int(d)), idx
        assert d < 0
        tour = oracle.apply(tour, int(i), int(j))
        L += int(d)
    assert np.array_equal(tour, res["tour"]) and L == res["length"] == oracle.tour_length(c, tour)
    assert oracle.pruned_best_move(c, tour, K, nbr=nb) == (0, 1, 0)
    assert full["length"] <= res["length"]
    assert full["length"] == oracle.tour_length(c, full["tour"])
    assert oracle.best_move(c, full["tour"]) == (0, 1, 0)
