"""Execution switches that must not change any result: CUDA-graph batches on
and off, and the pruned sweep's threads per position (read per launch)."""
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
