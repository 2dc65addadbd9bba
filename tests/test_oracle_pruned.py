"""Pins for the oracle's neighbourhood-pruned 2-opt (
L18 §V "Possibly limiting the neighborhood would also bring an improvement in
efficiency", L26 §VII "neighborhood pruning"; reading R18).

Independent references (none calls the oracle's arithmetic):
  * py_knn: every other city sorted by (nint distance, id) with the integer
    closed form nint(sqrt(s)) = (isqrt(4s)+1)//2;
  * brute-force neighbourhood: each 2-opt neighbour is built by explicit list
    reversal; the edges it CREATES are found by comparing the two undirected
    edge sets (no position formula), its length change by full recomputation;
  * K >= n-1 must reduce to the full neighbourhood, i.e. the plain oracle;
  * the list enumeration must equal the plain membership scan.
"""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs
from tests.test_oracle import np_dist_matrix, py_dist, py_length


def py_knn(coords, K):
    n = len(coords)
    out = []
    for a in range(n):
        others = sorted((py_dist(coords[a], coords[c]), c) for c in range(n) if c != a)
        row = [c for _, c in others[:K]]
        out.append(row + [-1] * (K - len(row)))
    return out


def candidate_edges(nbr):
    E = set()
    for a, row in enumerate(nbr):
        for c in row:
            if c >= 0:
                E.add(frozenset((a, c)))
    return E


def edge_set(tour):
    n = len(tour)
    return {frozenset((tour[k], tour[(k + 1) % n])) for k in range(n)}


def brute_pruned_best(coords, tour, K):
    """Lowest (dL, Fig. 3 cell) over the 2-opt neighbours that create an edge of E_K."""
    coords = [tuple(map(int, c)) for c in coords]
    tour = [int(c) for c in tour]
    n = len(tour)
    E = candidate_edges(py_knn(coords, K))
    L0 = py_length(coords, tour)
    old = edge_set(tour)
    best = (0, 0, 0, 1)  # (dL, cell, i, j): the seed pair (0, 1) of reading R7
    for j in range(1, n):
        for i in range(j):
            t2 = tour[: i + 1] + tour[i + 1 : j + 1][::-1] + tour[j + 1 :]
            created = edge_set(t2) - old
            if not (created & E):
                continue
            dL = py_length(coords, t2) - L0
            if dL < 0:
                best = min(best, (dL, j * (j - 1) // 2 + i, i, j))
    return best[2], best[3], best[0]


def _instances():
    out = []
    for n in (3, 4, 5, 6, 8, 11, 14):
        for seed in (1, 2):
            out.append((f"uniform-{n}-{seed}", inputs.make_coords("uniform", n, seed), inputs.random_tour(n, seed)))
    out.append(("lattice-16", inputs.make_coords("lattice", 16, 3), inputs.random_tour(16, 3)))
    grid = np.array([[x * 100, y * 100] for x in range(4) for y in range(4)], dtype=np.int32)  # ties everywhere
    out.append(("grid-4x4", grid, inputs.random_tour(16, 5)))
    dup = inputs.make_coords("uniform", 12, 4)
    dup[5] = dup[2]
    dup[9] = dup[2]  # duplicate cities: d = 0
    out.append(("duplicates-12", dup, inputs.random_tour(12, 4)))
    line = np.array([[37 * k % 1000, 500] for k in range(13)], dtype=np.int32)  # collinear
    out.append(("collinear-13", line, inputs.random_tour(13, 6)))
    return out


@pytest.mark.parametrize("name,coords,tour", _instances(), ids=lambda v: v if isinstance(v, str) else "")
def test_knn_matches_sorted_definition(name, coords, tour):
    n = len(coords)
    for K in (1, 2, 3, n - 1, n + 2):
        assert oracle.knn(coords, K).tolist() == py_knn(coords.tolist(), K), K


@pytest.mark.parametrize("name,coords,tour", _instances(), ids=lambda v: v if isinstance(v, str) else "")
def test_pruned_best_move_brute_force(name, coords, tour):
    n = len(coords)
    for K in (1, 2, 3, 5, n - 1):
        want = brute_pruned_best(coords, tour, K)
        assert oracle.pruned_best_move(coords, tour, K, plain=True) == want, K
        assert oracle.pruned_best_move(coords, tour, K) == want, K


@pytest.mark.parametrize("kind,n,seed", [("uniform", 60, 1), ("uniform", 97, 2), ("lattice", 80, 1)])
def test_full_K_is_the_full_neighbourhood(kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    assert oracle.pruned_best_move(c, t, n - 1) == oracle.best_move(c, t)
    a = oracle.pruned_local_search(c, t, n - 1, trace_cap=10_000)
    b = oracle.local_search(c, t, trace_cap=10_000)
    assert a["length"] == b["length"] and a["iterations"] == b["iterations"]
    assert np.array_equal(a["tour"], b["tour"]) and np.array_equal(a["trace"], b["trace"])


@pytest.mark.parametrize("kind,n,seed", [("uniform", 150, 1), ("lattice", 200, 2), ("uniform", 257, 3)])
def test_list_enumeration_equals_plain_scan(kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    tours = [inputs.random_tour(n, seed), inputs.hilbert_tour(c)]
    mid = oracle.local_search(c, inputs.random_tour(n, seed + 7), max_iters=n // 3)["tour"]
    tours.append(mid)
    for t in tours:
        for K in (1, 2, 4, 7, 8, 16):
            nb = oracle.knn(c, K)
            assert oracle.pruned_best_move(c, t, K, nbr=nb) == oracle.pruned_best_move(c, t, K, plain=True, nbr=nb)


@pytest.mark.parametrize("kind,n,seed,K", [("uniform", 120, 1, 4), ("lattice", 150, 2, 8), ("uniform", 200, 3, 2)])
def test_pruned_local_search_invariants(kind, n, seed, K):
    c = inputs.make_coords(kind, n, seed)
    t0 = inputs.random_tour(n, seed)
    res = oracle.pruned_local_search(c, t0, K, trace_cap=100_000)
    plain = oracle.pruned_local_search(c, t0, K, trace_cap=100_000, plain=True)
    assert np.array_equal(res["trace"], plain["trace"]) and np.array_equal(res["tour"], plain["tour"])
    assert res["status"] == 0
    # replay: every traced delta equals the recomputed length change, and it is
    # the best candidate move of the brute-force pruned neighbourhood (n <= 120)
    t = [int(x) for x in t0]
    L = py_length(c.tolist(), t)
    E = candidate_edges(py_knn(c.tolist(), K))
    for step, (i, j, d) in enumerate(res["trace"].tolist()):
        t2 = t[: i + 1] + t[i + 1 : j + 1][::-1] + t[j + 1 :]
        assert edge_set(t2) - edge_set(t) & E
        L2 = py_length(c.tolist(), t2)
        assert L2 - L == d < 0
        if n <= 120 and step % 25 == 0:
            assert brute_pruned_best(c, t, K) == (i, j, d)
        t, L = t2, L2
    assert L == res["length"] and t == res["tour"].tolist()
    assert sorted(t) == list(range(n)) and t[0] == t0[0]
    # certificate: no pair of M_K improves the final tour (vectorised membership)
    P = np.asarray(c)[np.r_[t, t[:1]]]
    D = np_dist_matrix(P)
    e = np.array([D[k, k + 1] for k in range(n)])
    ii, jj = np.triu_indices(n, k=1)
    delta = D[ii, jj] + D[ii + 1, jj + 1] - e[ii] - e[jj]
    nb = np.array(py_knn(c.tolist(), K))
    A = np.zeros((n, n), dtype=bool)
    for a in range(n):
        for x in nb[a]:
            if x >= 0:
                A[a, x] = A[x, a] = True
    tt = np.array(t + t[:1])
    member = A[tt[ii], tt[jj]] | A[tt[ii + 1], tt[jj + 1]]
    assert not np.any(delta[member] < 0)
    # pruning can only stop early: continuing with the full neighbourhood from
    # the pruned minimum reaches a full 2-opt local minimum at least as short
    full = oracle.local_search(c, res["tour"])
    assert full["length"] <= res["length"]
    assert oracle.best_move(c, full["tour"])[2] == 0


def test_pruned_max_iters_status():
    c = inputs.make_coords("uniform", 100, 4)
    t = inputs.random_tour(100, 4)
    full = oracle.pruned_local_search(c, t, 5)
    for cap in (0, 1, 7):
        r = oracle.pruned_local_search(c, t, 5, max_iters=cap)
        assert r["iterations"] == cap and r["status"] == 1
    r = oracle.pruned_local_search(c, t, 5, max_iters=full["iterations"])
    assert r["status"] == 0 and r["length"] == full["length"]


def brute_pruned_first(coords, tour, K):
    """First 2-opt neighbour in cell order that creates an edge of E_K and shortens the tour."""
    coords = [tuple(map(int, c)) for c in coords]
    tour = [int(c) for c in tour]
    n = len(tour)
    E = candidate_edges(py_knn(coords, K))
    L0 = py_length(coords, tour)
    old = edge_set(tour)
    for j in range(1, n):
        for i in range(j):
            t2 = tour[: i + 1] + tour[i + 1 : j + 1][::-1] + tour[j + 1 :]
            if (edge_set(t2) - old) & E and py_length(coords, t2) - L0 < 0:
                return i, j, py_length(coords, t2) - L0
    return 0, 1, 0


@pytest.mark.parametrize("name,coords,tour", _instances(), ids=lambda v: v if isinstance(v, str) else "")
def test_pruned_first_move_brute_force(name, coords, tour):
    n = len(coords)
    for K in (1, 2, 3, 5, n - 1):
        assert oracle.pruned_first_move(coords, tour, K) == brute_pruned_first(coords, tour, K), K
    assert oracle.pruned_first_move(coords, tour, max(1, n - 1)) == oracle.first_move(coords, tour)


@pytest.mark.parametrize("kind,n,seed,K", [("uniform", 80, 1, 4), ("lattice", 120, 2, 8)])
def test_pruned_first_local_search(kind, n, seed, K):
    c = inputs.make_coords(kind, n, seed)
    t0 = inputs.random_tour(n, seed)
    res = oracle.pruned_local_search(c, t0, K, trace_cap=100_000, first=True)
    t = [int(x) for x in t0]
    for step, (i, j, d) in enumerate(res["trace"].tolist()):
        if step % 10 == 0:
            assert brute_pruned_first(c, t, K) == (i, j, d)
        t = t[: i + 1] + t[i + 1 : j + 1][::-1] + t[j + 1 :]
    assert t == res["tour"].tolist()
    assert oracle.pruned_best_move(c, res["tour"], K) == (0, 1, 0)  # the same M_K local minimum certificate
    full = oracle.pruned_local_search(c, t0, n - 1, first=True)
    assert full["length"] == oracle.first_local_search(c, t0)["length"]
