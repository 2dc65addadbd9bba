"""GPU parity of first-improvement 2-opt (TSP2OPT_OPT_FIRST_IMPROVEMENT;
SURVEY.md §8(f) NEXT-4; reading R20: the improving pair with the
lowest Fig. 3 cell) against oracle.first_* -- bit-exact per sweep and per
traced move, through the C ABI."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


def _handle(c):
    g = tsp2opt.TSP2Opt(c)
    g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
    return g


@pytest.mark.parametrize("n", [3, 4, 5, 7, 16, 33, 100, 481, 1002, 2500])
@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_first_move_parity(gpu, n, kind):
    c = inputs.make_coords(kind, n, 9)
    mid = oracle.local_search(c, inputs.random_tour(n, 10), max_iters=n)["tour"]  # few improving pairs left
    with _handle(c) as g:
        for t in (inputs.random_tour(n, 9), inputs.hilbert_tour(c), mid):
            assert g.best_move(t) == oracle.first_move(c, t)


@pytest.mark.parametrize("bounds", ["0", "1", "2", "3"])
@pytest.mark.parametrize("rows", [7, 15])
@pytest.mark.parametrize("warps,tj", [(1, 2), (1, 3), (1, 32), (2, 64), (4, 128), (3, 7)])
def test_first_move_geometries(gpu, monkeypatch, rows, warps, tj, bounds):
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    monkeypatch.setenv("TSP2OPT_ROWS", str(rows))
    monkeypatch.setenv("TSP2OPT_CULL_ROWS", str(rows))
    monkeypatch.setenv("TSP2OPT_WARPS", str(warps))
    monkeypatch.setenv("TSP2OPT_TJ", str(tj))
    for kind, n in (("uniform", 300), ("lattice", 961)):
        c = inputs.make_coords(kind, n, 4)
        mid = oracle.local_search(c, inputs.random_tour(n, 5), max_iters=n)["tour"]
        with _handle(c) as g:
            for t in (inputs.random_tour(n, 4), inputs.hilbert_tour(c), mid):
                assert g.best_move(t) == oracle.first_move(c, t)


@pytest.mark.parametrize("bounds", ["1", "3"])
@pytest.mark.parametrize("kind,n,seed,cap", [("uniform", 100, 1, -1), ("lattice", 100, 2, -1),
                                             ("uniform", 300, 3, -1), ("lattice", 500, 4, -1),
                                             ("uniform", 1002, 5, 3000), ("lattice", 2000, 6, 1500)])
def test_first_local_search_trace(gpu, monkeypatch, bounds, kind, n, seed, cap):
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    want = oracle.first_local_search(c, t, max_iters=cap, trace_cap=10 * n)
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, 10 * n)
        res = g.local_search(t, max_iters=None if cap < 0 else cap)
        trace = g.get_trace(10 * n)
    assert res["status"] == want["status"]
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
    assert np.array_equal(res["tour"], want["tour"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), want["trace"])


@pytest.mark.parametrize("bounds", ["1", "3"])
def test_first_mixed_operations(gpu, monkeypatch, bounds):
    """Explicit applies, switching the rule off and on around device-side
    iterations, a new tour, simulated shards (the min over shards by cell),
    and the exclusive options."""
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    n = 1500
    c = inputs.make_coords("lattice", n, 7)
    t = inputs.random_tour(n, 7)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_tour(t)
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
        cur = t.copy()
        assert g.best_move() == oracle.first_move(c, cur)
        for i, j in ((0, 1), (3, 900), (0, n - 1), (n - 2, n - 1), (200, 1400)):
            g.apply(i, j)
            cur = oracle.apply(cur, i, j)
            assert g.best_move() == oracle.first_move(c, cur)
        g.iterate_async(7)
        g.sync()
        for _ in range(7):
            i, j, d = oracle.first_move(c, cur)
            cur = oracle.apply(cur, i, j)
        assert np.array_equal(g.get_tour()[0], cur)
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 0)  # best improvement on the same tour
        g.iterate_async(4)
        g.sync()
        for _ in range(4):
            i, j, d = oracle.best_move(c, cur)
            cur = oracle.apply(cur, i, j)
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
        g.iterate_async(5)  # no best_move first: the pending key must not leak across rules
        g.sync()
        for _ in range(5):
            i, j, d = oracle.first_move(c, cur)
            cur = oracle.apply(cur, i, j)
        tour, L = g.get_tour()
        assert np.array_equal(tour, cur) and L == oracle.tour_length(c, cur)
        want = oracle.first_move(c, cur)
        for world in (2, 3, 8):  # each shard's first improving pair; the lowest cell wins
            keys = []
            for r in range(world):
                g.debug_set_shard(r, world)
                i, j, d = g.best_move()
                if d < 0:
                    keys.append((j * (j - 1) // 2 + i, i, j, d))
            g.debug_set_shard(0, 1)
            _, i, j, d = min(keys)
            assert (i, j, d) == want, world
        with pytest.raises(tsp2opt.TSP2OptError):
            g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)


@pytest.mark.parametrize("cfg,nsamples", [("C3", 6), ("C4", 4), ("C5", 2)])
def test_first_full_size_from_mf(gpu, cfg, nsamples):
    """At BASELINE.json sizes from the Multiple Fragment start, first
    improvement to the local minimum in the default launch configuration:
    trace replay, sampled oracle re-checks, and the 2-opt certificate."""
    c, _ = inputs.config_instance(cfg, "random")
    n = len(c)
    cap = 20 * n
    with _handle(c) as g:
        t = g.mf_tour()["tour"]
        g.set_option(tsp2opt.OPT_TRACE, cap)
        res = g.local_search(t)
        trace = g.get_trace(cap)
    k = res["iterations"]
    assert res["status"] == tsp2opt.OK and len(trace) == k > 0
    picks = set(np.linspace(0, k - 1, nsamples).astype(int).tolist())
    tour = t.copy()
    L = oracle.tour_length(c, tour)
    for idx, (i, j, d) in enumerate(trace.tolist()):
        if idx in picks:
            assert oracle.first_move(c, tour) == (i, j, d), idx
        assert d < 0
        tour = oracle.apply(tour, i, j)
        L += d
    assert np.array_equal(tour, res["tour"]) and L == res["length"] == oracle.tour_length(c, tour)
    assert oracle.best_move(c, res["tour"]) == (0, 1, 0)


@pytest.mark.parametrize("n", [5, 33, 481, 2500])
@pytest.mark.parametrize("K", [1, 4, 8, 16])
def test_pruned_first_move_parity(gpu, n, K):
    """First improvement over the pruned neighbourhood M_K (readings R18 + R20)."""
    c = inputs.make_coords("lattice" if n % 2 else "uniform", n, 3)
    nb = oracle.knn(c, K)
    mid = oracle.local_search(c, inputs.random_tour(n, 4), max_iters=n)["tour"]
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
        for t in (inputs.random_tour(n, 3), inputs.hilbert_tour(c), mid):
            assert g.best_move(t) == oracle.pruned_first_move(c, t, K, nbr=nb)


@pytest.mark.parametrize("kind,n,seed,K,cap", [("uniform", 200, 1, 4, -1), ("lattice", 500, 2, 8, -1),
                                               ("uniform", 1002, 3, 16, 2000)])
def test_pruned_first_local_search(gpu, kind, n, seed, K, cap):
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    want = oracle.pruned_local_search(c, t, K, first=True, max_iters=cap, trace_cap=40 * n)
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
        g.set_option(tsp2opt.OPT_TRACE, 40 * n)
        res = g.local_search(t, max_iters=None if cap < 0 else cap)
        trace = g.get_trace(40 * n)
    assert res["status"] == want["status"]
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
    assert np.array_equal(res["tour"], want["tour"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), want["trace"])
