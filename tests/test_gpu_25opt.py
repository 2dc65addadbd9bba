"""GPU parity of best-improvement 2.5-opt (TSP2OPT_OPT_NODE_INSERTION; SURVEY.md
§8(f) NEXT-4; L26 §VII; reading R19) against oracle.*25 --
bit-exact: (i, j, type, delta) per sweep, the traced moves, final tour,
length and move count, through the C ABI."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu

SIZES = [3, 4, 5, 7, 16, 33, 100, 481, 1002, 2500]


def _handle(c):
    g = tsp2opt.TSP2Opt(c)
    g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
    return g


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_best_move25_parity(gpu, n, kind):
    c = inputs.make_coords(kind, n, 7)
    with _handle(c) as g:
        for t in (inputs.random_tour(n, 7), inputs.random_tour(n, 8), inputs.hilbert_tour(c)):
            assert g.best_move_typed(t) == oracle.best_move25(c, t)
            i, j, typ, d = oracle.best_move25(c, t)
            assert g.best_move(t) == (i, j, d)


@pytest.mark.parametrize("bounds", ["0", "1", "2", "3"])
@pytest.mark.parametrize("warps,tj", [(1, 2), (1, 3), (1, 32), (2, 64), (4, 128), (3, 7)])
def test_best_move25_geometries(gpu, monkeypatch, warps, tj, bounds):
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    monkeypatch.setenv("TSP2OPT_WARPS", str(warps))
    monkeypatch.setenv("TSP2OPT_TJ", str(tj))
    for kind, n in (("uniform", 257), ("lattice", 700)):
        c = inputs.make_coords(kind, n, 3)
        with _handle(c) as g:
            for t in (inputs.random_tour(n, 3), inputs.hilbert_tour(c)):
                assert g.best_move_typed(t) == oracle.best_move25(c, t)
            # mid-search tours: few candidates, ties among small deltas
            t = oracle.local_search25(c, inputs.random_tour(n, 4), max_iters=n // 2)["tour"]
            assert g.best_move_typed(t) == oracle.best_move25(c, t)


@pytest.mark.parametrize("kind,n,seed", [("uniform", 100, 1), ("lattice", 100, 2), ("uniform", 1002, 2),
                                         ("lattice", 1002, 1), ("uniform", 2000, 3)])
def test_local_search25_trace(gpu, kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    cap = 10 * n
    want = oracle.local_search25(c, t, trace_cap=cap)
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, cap)
        res = g.local_search(t)
        trace = g.get_trace_typed(cap)
    assert res["status"] == want["status"] == tsp2opt.OK
    assert res["iterations"] == want["iterations"] and res["length"] == want["length"]
    assert np.array_equal(res["tour"], want["tour"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), want["trace"])
    assert set(np.unique(want["trace"][:, 3]).tolist()) == {0, 1, 2}  # every move type occurs


@pytest.mark.parametrize("bounds", ["2", "3"])
@pytest.mark.parametrize("cull_tj", ["2", "3", "32", "64"])
@pytest.mark.parametrize("kind,n,seed", [("uniform", 1002, 5), ("lattice", 2000, 6)])
def test_local_search25_culled(gpu, monkeypatch, cull_tj, kind, n, seed, bounds):
    """The pre-sweep cull with the gain term (box + cull + list sweep), forced at
    small n, with narrow and ragged column chunks; bounds 3 keeps the tiles'
    own minima and re-sweeps only the tiles the last move touched."""
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    monkeypatch.setenv("TSP2OPT_CULL_TJ", cull_tj)
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    want = oracle.local_search25(c, t, trace_cap=10 * n)
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, 10 * n)
        res = g.local_search(t)
        trace = g.get_trace_typed(10 * n)
        assert g.best_move_typed(inputs.hilbert_tour(c)) == oracle.best_move25(c, inputs.hilbert_tour(c))
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
    assert np.array_equal(res["tour"], want["tour"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), want["trace"])


def test_local_search25_ties_and_degenerate(gpu):
    grid = np.array([[x * 300, y * 300] for x in range(20) for y in range(15)], dtype=np.int32)
    dup = inputs.make_coords("uniform", 200, 9)
    dup[50:60] = dup[7]
    line = np.array([[(97 * k) % 30000, 12345] for k in range(150)], dtype=np.int32)
    for c in (grid, dup, line, inputs.make_coords("uniform", 3, 1), inputs.make_coords("uniform", 4, 2),
              inputs.make_coords("uniform", 5, 3)):
        n = len(c)
        t = inputs.random_tour(n, 11)
        with _handle(c) as g:
            res = g.local_search(t)
        want = oracle.local_search25(c, t)
        assert (res["length"], res["iterations"]) == (want["length"], want["iterations"])
        assert np.array_equal(res["tour"], want["tour"])


def test_local_search25_max_iters(gpu):
    c = inputs.make_coords("uniform", 1002, 4)
    t = inputs.random_tour(1002, 4)
    with _handle(c) as g:
        for cap in (0, 1, 7, 100):
            res = g.local_search(t, max_iters=cap)
            want = oracle.local_search25(c, t, max_iters=cap)
            assert res["status"] == want["status"] == tsp2opt.MAXITER
            assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
            assert np.array_equal(res["tour"], want["tour"])


@pytest.mark.parametrize("bounds", ["1", "3"])
def test_25opt_mixed_operations(gpu, monkeypatch, bounds):
    """Explicit moves of every type (edges of the position range included),
    switching the mode off and on around device-side iterations, simulated
    shards, and the error cases; bounds 3: stored tile minima across all of it."""
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    n = 1200
    c = inputs.make_coords("lattice", n, 5)
    t = inputs.random_tour(n, 5)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_tour(t)
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)  # gains built from the loaded tour
        cur = t.copy()
        L = oracle.tour_length(c, cur)
        assert g.best_move_typed() == oracle.best_move25(c, cur)
        for i, j, typ in ((0, 2, 1), (0, 2, 2), (0, n - 1, 1), (0, n - 1, 2), (5, 900, 1), (5, 900, 2),
                          (n - 3, n - 1, 1), (n - 3, n - 1, 2), (3, 4, 0), (0, n - 1, 0), (17, 1000, 0)):
            d = oracle.delta25(c, cur, i, j, typ)
            g.apply_typed(i, j, typ)
            cur = oracle.apply25(cur, i, j, typ)
            L += d
            tour, length = g.get_tour()
            assert np.array_equal(tour, cur) and length == L == oracle.tour_length(c, cur)
            assert g.best_move_typed() == oracle.best_move25(c, cur)
        for bad in ((5, 6, 1), (5, 6, 2), (6, 5, 1), (0, n, 2), (0, 5, 3)):
            with pytest.raises(tsp2opt.TSP2OptError):
                g.apply_typed(*bad)
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 0)  # 2-opt on the same tour, gains not maintained
        assert g.best_move() == oracle.best_move(c, cur)
        g.iterate_async(6)
        g.sync()
        for _ in range(6):
            i, j, d = oracle.best_move(c, cur)
            cur = oracle.apply(cur, i, j)
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)  # gains rebuilt; no best_move before the loop
        g.iterate_async(9)
        g.sync()
        for _ in range(9):
            i, j, typ, d = oracle.best_move25(c, cur)
            cur = oracle.apply25(cur, i, j, typ)
        assert np.array_equal(g.get_tour()[0], cur)
        want = oracle.best_move25(c, cur)
        for world in (2, 3, 8):  # min over simulated shards of the tile list
            keys = []
            for r in range(world):
                g.debug_set_shard(r, world)
                i, j, d = g.best_move()
                keys.append((d, j * (j - 1) // 2 + i, i, j))
            d, _, i, j = min(keys)
            assert (i, j, d) == (want[0], want[1], want[3]), world
        g.debug_set_shard(0, 1)
        with pytest.raises(tsp2opt.TSP2OptError):
            g.set_option(tsp2opt.OPT_NEIGHBOURS, 8)  # exclusive modes


@pytest.mark.parametrize("cfg,nsamples", [("C3", 4), ("C4", 3), ("C5", 2)])
def test_local_search25_full_size_from_mf(gpu, cfg, nsamples):
    """At BASELINE.json sizes from the Multiple Fragment start: the typed move
    trace replayed on the CPU gives the final tour and length; sampled
    iterations (first, last, evenly spaced) re-swept by the oracle give the
    traced move; the final tour carries the oracle's 2.5-opt certificate."""
    c, _ = inputs.config_instance(cfg, "random")
    n = len(c)
    cap = 4 * n
    with _handle(c) as g:
        t = g.mf_tour()["tour"]
        g.set_option(tsp2opt.OPT_TRACE, cap)
        res = g.local_search(t)
        trace = g.get_trace_typed(cap)
    k = res["iterations"]
    assert res["status"] == tsp2opt.OK and len(trace) == k > 0
    picks = set(np.linspace(0, k - 1, nsamples).astype(int).tolist())
    tour = t.copy()
    L = oracle.tour_length(c, tour)
    for idx, (i, j, d, typ) in enumerate(trace.tolist()):
        if idx in picks:
            assert oracle.best_move25(c, tour) == (i, j, typ, d), idx
        assert d < 0
        tour = oracle.apply25(tour, i, j, typ)
        L += d
    assert np.array_equal(tour, res["tour"]) and L == res["length"] == oracle.tour_length(c, tour)
    assert oracle.best_move25(c, res["tour"]) == (0, 1, 0, 0)
