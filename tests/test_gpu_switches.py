"""Execution switches that must not change any result: CUDA-graph batches on
and off, and the pruned sweep's threads per position (read per launch)."""
import functools

import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("graph", ["0", "1"])
@pytest.mark.parametrize("mode", ["cull3", "pruned", "first", "or25"])
def test_graph_switch(gpu, monkeypatch, graph, mode):
    monkeypatch.setenv("TSP2OPT_GRAPH", graph)
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", "3")
    n = 2000
    c = inputs.make_coords("lattice", n, 21)
    t = inputs.hilbert_tour(c)
    with tsp2opt.TSP2Opt(c) as g:
        if mode == "pruned":
            g.set_option(tsp2opt.OPT_NEIGHBOURS, 8)
            want = oracle.pruned_local_search(c, t, 8)
        elif mode == "first":
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
            want = oracle.first_local_search(c, t)
        elif mode == "or25":
            g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
            want = oracle.local_search25(c, t)
        else:
            want = oracle.local_search(c, t)
        res = g.local_search(t)
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
    assert np.array_equal(res["tour"], want["tour"])
    assert res["iterations"] > 64  # at least one full graph batch


@pytest.mark.parametrize("tp", ["1", "2", "4", "8"])
def test_pruned_threads_per_position(gpu, monkeypatch, tp):
    monkeypatch.setenv("TSP2OPT_PRUNED_TP", tp)
    n = 3000
    c = inputs.make_coords("uniform", n, 22)
    t = inputs.random_tour(n, 22)
    with tsp2opt.TSP2Opt(c) as g:
        for K in (3, 16):
            g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
            assert g.best_move(t) == oracle.pruned_best_move(c, t, K)
        res = g.local_search(t)
    want = oracle.pruned_local_search(c, t, 16)
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])


@pytest.mark.parametrize("kind,n,seed", [("uniform", 1002, 31), ("lattice", 3001, 32)])
def test_global_seed_switch(gpu, monkeypatch, kind, n, seed):
    """TSP2OPT_GLOBAL_SEED=1: each dense sweep starts from the best tile minimum
    of the previous sweep that the applied reversal leaves intact."""
    monkeypatch.setenv("TSP2OPT_GLOBAL_SEED", "1")
    monkeypatch.setenv("TSP2OPT_PERSISTENT", "0")
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    want = oracle.local_search(c, t, trace_cap=10 * n)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, 10 * n)
        res = g.local_search(t)
        trace = g.get_trace(10 * n)
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), want["trace"])


@functools.lru_cache(maxsize=None)
def _inc_case(first, start, cap):
    c = inputs.make_coords("lattice", 1500, 5)  # 7 row blocks x 94 chunks: two groups of minima
    t = inputs.make_tour(start, c, 3)
    ls = oracle.first_local_search if first else oracle.local_search
    return c, t, ls(c, t, max_iters=cap, trace_cap=20000)


@pytest.mark.parametrize("barriers,part", [("1", "1"), ("1", "4"), ("1", "16"), ("2", "1"), ("2", "2"), ("2", "4"),
                                           ("2", "16"), ("3", "0"), ("3", "4")])
@pytest.mark.parametrize("first", [0, 1])
@pytest.mark.parametrize("start,cap", [("hilbert", -1), ("random", 400)])
def test_incremental_persistent_variants(gpu, monkeypatch, barriers, part, first, start, cap):
    """The persistent incremental search (TSP2OPT_OPT_TILE_BOUNDS = 3): one barrier per move (the dirty
    tiles swept from the pre-move state through the mirror map, conservative boxes), two with the
    out-of-place apply and group minima, or three with the in-place apply; kept tiles split into column
    parts of 1 / 2 / 4 / 16 columns or swept whole -- every move equal to the oracle's, with a move cap
    that ends a search mid-way (the alternate buffer copied back) and (best improvement) a resumed search
    after it.  (The first-improvement oracle from a random tour to the minimum takes minutes: capped only.)"""
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", "3")
    monkeypatch.setenv("TSP2OPT_CULL_TJ", "16")
    monkeypatch.setenv("TSP2OPT_INC_BARRIERS", barriers)
    monkeypatch.setenv("TSP2OPT_INC_PART", part)
    c, t, want = _inc_case(first, start, cap)
    with tsp2opt.TSP2Opt(c) as g:
        if first:
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
        g.set_option(tsp2opt.OPT_TRACE, 20000)
        res = g.local_search(t, max_iters=None if cap < 0 else cap)
        got = np.asarray(g.get_trace(20000), dtype=np.int64)
        assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
        assert np.array_equal(res["tour"], want["tour"])
        assert np.array_equal(got, want["trace"][: len(got)]) and len(got) == want["iterations"]
        assert np.array_equal(g.get_tour()[0], want["tour"])
        if cap > 0 and not first:  # resume to the local minimum from the capped state
            full = _inc_case(first, start, -1)[2]
            r2 = g.local_search_current()
            assert res["iterations"] + r2["iterations"] == full["iterations"]
            assert r2["length"] == full["length"]
            assert np.array_equal(g.get_tour()[0], full["tour"])
