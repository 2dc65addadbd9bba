"""Pins for the oracle's first-improvement 2-opt (
DESIGN.md reading R20: the improving pair with the lowest Fig. 3 cell).

Independent references: every neighbour built by explicit list reversal in
the Fig. 3 cell order with its length recomputed from scratch (brute force);
the best-improvement oracle as a local-minimum certificate."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs
from tests.test_oracle import brute_neighbours, py_length


def brute_first(coords, tour):
    for dL, cell, i, j, _ in brute_neighbours(coords, tour):  # j-major, i ascending: cell order
        if dL < 0:
            return i, j, dL
    return 0, 1, 0


@pytest.mark.parametrize("kind,n,seed", [("uniform", 3, 1), ("uniform", 4, 2), ("uniform", 7, 3), ("uniform", 12, 4),
                                         ("lattice", 16, 5), ("uniform", 30, 6)])
def test_first_move_brute_force(kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    for t in (inputs.random_tour(n, seed), inputs.random_tour(n, seed + 1), inputs.hilbert_tour(c)):
        assert oracle.first_move(c, t) == brute_first(c.tolist(), list(t))


@pytest.mark.parametrize("kind,n,seed", [("uniform", 40, 1), ("lattice", 60, 2), ("uniform", 100, 3)])
def test_first_local_search_invariants(kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    t0 = inputs.random_tour(n, seed)
    res = oracle.first_local_search(c, t0, trace_cap=100_000)
    assert res["status"] == 0
    t = [int(x) for x in t0]
    L = py_length(c.tolist(), t)
    for step, (i, j, d) in enumerate(res["trace"].tolist()):
        if n <= 40 or step % 20 == 0:
            assert brute_first(c.tolist(), t) == (i, j, d)
        t2 = t[: i + 1] + t[i + 1 : j + 1][::-1] + t[j + 1 :]
        L2 = py_length(c.tolist(), t2)
        assert L2 - L == d < 0
        t, L = t2, L2
    assert t == res["tour"].tolist() and L == res["length"]
    assert oracle.best_move(c, res["tour"]) == (0, 1, 0)  # a 2-opt local minimum


def test_first_max_iters_status():
    c = inputs.make_coords("uniform", 100, 4)
    t = inputs.random_tour(100, 4)
    full = oracle.first_local_search(c, t)
    for cap in (0, 1, 7):
        r = oracle.first_local_search(c, t, max_iters=cap)
        assert r["iterations"] == cap and r["status"] == 1
    r = oracle.first_local_search(c, t, max_iters=full["iterations"])
    assert r["status"] == 0 and r["length"] == full["length"]
