"""Pins for the oracle's Iterated Local Search (L10 Algorithm 1; readings R14-R16)."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs
from tests.test_oracle import np_best_move, py_length


def py_cuts(n, seed, it):
    m = max(1, (n - 1) // 3)
    r = inputs.splitmix64(seed, 3, offset=3 * it)  # Vigna-pinned generator (tests/test_inputs.py)
    l0, l1, l2 = (1 + int(x % np.uint64(m)) for x in r)
    return l0, l0 + l1, l0 + l1 + l2


def py_local_search(coords, tour):
    t = np.array(tour)
    while True:
        i, j, d, *_ = np_best_move(coords, t)
        if d >= 0:
            return t
        t = np.concatenate([t[: i + 1], t[i + 1 : j + 1][::-1], t[j + 1 :]])


@pytest.mark.parametrize("n,seed", [(8, 1), (50, 2), (1002, 7), (85900, 3)])
def test_double_bridge_cuts_match_generator(n, seed):
    for it in (0, 1, 5, 1000):
        a, b, c = oracle.double_bridge_cuts(n, seed, it)
        assert (a, b, c) == py_cuts(n, seed, it)
        assert 1 <= a < b < c <= n - 1


def test_double_bridge_is_acbd():
    rng = np.random.default_rng(0)
    for n in (8, 9, 30, 101):
        t = rng.permutation(n).astype(np.int32)
        for _ in range(5):
            a, b, c = sorted(rng.choice(np.arange(1, n), 3, replace=False).tolist())
            got = oracle.double_bridge(t, a, b, c)
            want = np.concatenate([t[:a], t[b:c], t[a:b], t[c:]])
            assert np.array_equal(got, want) and got[0] == t[0]
            # only the three edges (a-1,a), (b-1,b), (c-1,c) can be replaced
            old = {frozenset((t[k], t[(k + 1) % n])) for k in range(n)}
            new = {frozenset((got[k], got[(k + 1) % n])) for k in range(n)}
            assert len(old - new) == len(new - old) <= 3  # (fewer when a segment has one city)


@pytest.mark.parametrize("n,seed", [(12, 1), (16, 2), (20, 3)])
def test_ils_matches_independent_python(n, seed):
    coords = inputs.uniform_coords(n, seed)
    t0 = inputs.random_tour(n, seed)
    res = oracle.ils(coords, t0, 15, seed=99)
    best = py_local_search(coords, t0)
    L = py_length(coords, best)
    lengths = [L]
    for it in range(15):
        a, b, c = py_cuts(n, 99, it)
        cand = np.concatenate([best[:a], best[b:c], best[a:b], best[c:]])
        cand = py_local_search(coords, cand)
        if py_length(coords, cand) < L:
            best, L = cand, py_length(coords, cand)
        lengths.append(L)
    assert np.array_equal(res["tour"], best) and res["length"] == L
    assert res["lengths"].tolist() == lengths


def test_ils_invariants_medium():
    coords = inputs.uniform_coords(200, 5)
    t0 = inputs.random_tour(200, 5)
    res = oracle.ils(coords, t0, 30, seed=1)
    Ls = res["lengths"]
    assert (np.diff(Ls) <= 0).all() and Ls[-1] == res["length"] == oracle.tour_length(coords, res["tour"])
    assert oracle.best_move(coords, res["tour"])[2] == 0  # a 2-opt local minimum
    assert sorted(res["tour"].tolist()) == list(range(200)) and res["tour"][0] == t0[0]
    assert Ls[-1] <= oracle.local_search(coords, t0)["length"]


@pytest.mark.parametrize("kw", [dict(neighbours=6), dict(first=True), dict(neighbours=6, first=True),
                                dict(node_insertion=True)])
def test_ils_over_variants(kw):
    """ILS with another local search: the same perturbation / acceptance as a
    Python restatement of Algorithm 1 around the variant's oracle local search."""
    c = inputs.make_coords("uniform", 60, 5)
    t0 = inputs.random_tour(60, 5)

    def ls(t):
        if kw.get("node_insertion"):
            return oracle.local_search25(c, t)
        if kw.get("neighbours"):
            return oracle.pruned_local_search(c, t, kw["neighbours"], first=kw.get("first", False))
        return oracle.first_local_search(c, t)

    r = ls(t0)
    best, L = r["tour"], r["length"]
    lengths = [L]
    for it in range(6):
        a, b, cc = oracle.double_bridge_cuts(60, 99, it)
        r = ls(oracle.double_bridge(best, a, b, cc))
        if r["length"] < L:
            best, L = r["tour"], r["length"]
        lengths.append(L)
    got = oracle.ils(c, t0, 6, 99, **kw)
    assert got["length"] == L and np.array_equal(got["tour"], best)
    assert got["lengths"].tolist() == lengths
