"""Pins for the oracle's Multiple Fragment (greedy) start tour (L22 §V
"Multiple Fragment(Greedy) heuristic[18]"; reading R17).

The pins restate the definition independently of the oracle's sort + union-find
formulation: brute force repeatedly takes the globally smallest admissible edge
(both ends of degree < 2, no cycle -- checked by walking the partial path) with
distances from the integer closed form nint(sqrt(s)) = (isqrt(4s) + 1) // 2."""
import math

import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs


def nint_dist(a, b):
    s = int(a[0] - b[0]) ** 2 + int(a[1] - b[1]) ** 2
    return (math.isqrt(4 * s) + 1) // 2


def brute_mf(coords):
    n = len(coords)
    deg = [0] * n
    adj = [[] for _ in range(n)]

    def path_end(u):  # follow the partial path from an end u to its other end
        prev, cur = -1, u
        while True:
            nxt = [v for v in adj[cur] if v != prev]
            if not nxt:
                return cur
            prev, cur = cur, nxt[0]

    for _ in range(n - 1):
        best = None
        for u in range(n):
            for v in range(u + 1, n):
                if deg[u] < 2 and deg[v] < 2 and path_end(u) != v:
                    k = (nint_dist(coords[u], coords[v]), u, v)
                    best = k if best is None or k < best else best
        _, u, v = best
        adj[u].append(v), adj[v].append(u)
        deg[u] += 1
        deg[v] += 1
    a, b = [u for u in range(n) if deg[u] < 2]
    adj[a].append(b), adj[b].append(a)
    tour, prev, cur = [0], 0, min(adj[0])
    while cur != 0:
        tour.append(cur)
        prev, cur = cur, [v for v in adj[cur] if v != prev][0]
    return tour


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("kind,n", [("uniform", 3), ("uniform", 4), ("uniform", 9), ("uniform", 13),
                                    ("lattice", 12), ("lattice", 14)])
def test_mf_matches_brute_force_definition(kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    assert oracle.mf_tour(c).tolist() == brute_mf(c.tolist())


def test_mf_ties_small_grid():
    # a 3x4 unit grid: every candidate edge length ties with others, so the
    # (d, min id, max id) order decides everything
    c = np.array([[x * 1000, y * 1000] for y in range(3) for x in range(4)], dtype=np.int32)
    rng = np.random.default_rng(5)
    for _ in range(4):
        perm = rng.permutation(len(c))
        cc = c[perm]
        assert oracle.mf_tour(cc).tolist() == brute_mf(cc.tolist())


def test_mf_collinear_is_sorted_order():
    # distinct points on a line: every adjacent gap is shorter than any
    # non-adjacent edge, so greedy takes exactly the sorted path and closes it
    rng = np.random.default_rng(1)
    n = 300
    xs = np.sort(rng.choice(32000, n, replace=False))
    perm = rng.permutation(n)
    c = np.stack([xs[perm], np.full(n, 5)], axis=1).astype(np.int32)
    order = list(np.argsort(c[:, 0]))  # cities by x
    k = order.index(0)
    cyc = order[k:] + order[:k]
    if cyc[1] > cyc[-1]:
        cyc = [cyc[0]] + cyc[1:][::-1]
    assert oracle.mf_tour(c).tolist() == [int(v) for v in cyc]


@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_mf_tour_is_valid_and_short(kind):
    n = 2000
    c = inputs.make_coords(kind, n, 3)
    t = oracle.mf_tour(c)
    assert sorted(t.tolist()) == list(range(n)) and t[0] == 0 and t[1] < t[-1]
    # greedy is within a small factor of the 2-opt local minimum reached from it
    L = oracle.tour_length(c, t)
    assert L < oracle.tour_length(c, inputs.hilbert_tour(c))
    ls = oracle.local_search(c, t)
    assert ls["length"] <= L and L < 1.3 * ls["length"]


def test_mf_rejects_out_of_range():
    with pytest.raises(ValueError):
        oracle.mf_tour(np.zeros((2, 2), np.int32))
