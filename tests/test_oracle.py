"""Pins for the CPU oracle (oracle/) against things other than itself.

Independent references used here (none calls the oracle's own arithmetic):
  * py_nint(s) = (isqrt(4s)+1)//2  -- floor(sqrt(s)+1/2) = floor((floor(2 sqrt s)+1)/2)
    and floor(2 sqrt s) = isqrt(4s); Python's exact integer isqrt.
  * np_nint: float64 sqrt then floor(x+0.5); exact for s < 2^31 because sqrt(s) is
    never within 2.7e-6 of a half-integer there while the float64 error is < 1e-11.
  * explicit neighbour construction: each 2-opt neighbour is built by reversing the
    list slice and its length recomputed from scratch (no delta formula).
  * brute force over all (n-1)! tours for the global optimum (n <= 9).
"""
import itertools
import math
import os

import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def py_nint(s: int) -> int:
    return (math.isqrt(4 * s) + 1) // 2


def py_dist(a, b) -> int:
    dx = int(a[0]) - int(b[0])
    dy = int(a[1]) - int(b[1])
    return py_nint(dx * dx + dy * dy)


def py_length(coords, tour) -> int:
    n = len(tour)
    return sum(py_dist(coords[tour[k]], coords[tour[(k + 1) % n]]) for k in range(n))


def np_dist_matrix(P):
    P = np.asarray(P, dtype=np.int64)
    dx = P[:, None, 0] - P[None, :, 0]
    dy = P[:, None, 1] - P[None, :, 1]
    s = (dx * dx + dy * dy).astype(np.float64)
    return np.floor(np.sqrt(s) + 0.5).astype(np.int64)


def np_best_move(coords, tour):
    """Vectorised exhaustive sweep: all deltas, lowest delta then lowest Fig. 3 cell."""
    n = len(tour)
    P = np.asarray(coords)[np.r_[tour, tour[:1]]]
    D = np_dist_matrix(P)
    e = np.array([D[k, k + 1] for k in range(n)])
    i, j = np.triu_indices(n, k=1)  # i < j <= n-1
    d = D[i, j] + D[i + 1, j + 1] - e[i] - e[j]
    k = j * (j - 1) // 2 + i
    order = np.lexsort((k, d))
    b = order[0]
    return int(i[b]), int(j[b]), int(d[b]), d, i, j


def brute_neighbours(coords, tour):
    """Every 2-opt neighbour by explicit reversal, its exact length change."""
    n = len(tour)
    L0 = py_length(coords, tour)
    out = []
    for j in range(1, n):
        for i in range(j):
            t2 = list(tour[: i + 1]) + list(tour[i + 1 : j + 1])[::-1] + list(tour[j + 1 :])
            out.append((py_length(coords, t2) - L0, j * (j - 1) // 2 + i, i, j, t2))
    return out


# ----------------------------------------------------------------------------- distance

def test_nint_small_range_exhaustive():
    for s in range(0, 200_001):
        assert oracle.nint_sqrt(s) == py_nint(s)


def test_nint_boundaries_all_m():
    # every rounding boundary m^2-m, m^2-m+1, m^2+m, m^2+m+1 up to the max reachable s
    smax = 2 * 32767 * 32767
    for m in range(1, 46342):
        for s in (m * m - m, m * m - m + 1, m * m + m, m * m + m + 1, m * m):
            if 0 <= s <= smax:
                assert oracle.nint_sqrt(s) == py_nint(s), s
    assert oracle.nint_sqrt(smax) == py_nint(smax)


def test_nint_random_full_range():
    rng = np.random.default_rng(7)
    for s in rng.integers(0, 2 * 32767 * 32767 + 1, size=50_000):
        assert oracle.nint_sqrt(int(s)) == py_nint(int(s))


def test_dist_random_pairs_vs_python_and_float64():
    rng = np.random.default_rng(11)
    pts = rng.integers(0, 1 << 15, size=(20_000, 4))
    for x1, y1, x2, y2 in pts[:5000]:
        assert oracle.dist((x1, y1), (x2, y2)) == py_dist((x1, y1), (x2, y2))
    dx = (pts[:, 0] - pts[:, 2]).astype(np.int64)
    dy = (pts[:, 1] - pts[:, 3]).astype(np.int64)
    f64 = np.floor(np.sqrt((dx * dx + dy * dy).astype(np.float64)) + 0.5).astype(np.int64)
    py = np.array([py_nint(int(a * a + b * b)) for a, b in zip(dx, dy)])
    assert np.array_equal(f64, py)


def test_listing1_float_formula_is_not_exact():
    """Reading R3: Listing 1 (L16) `(int)(sqrtf(dx*dx+dy*dy)+0.5f)` in FP32 differs from
    the exact EUC_2D nint; the oracle follows the exact integer definition."""
    dx, dy = 28472, 28096
    s = dx * dx + dy * dy
    assert s == 40000 * 40000 + 40000  # just below the rounding boundary 40000.5^2
    exact = py_nint(s)
    f = np.float32(dx) * np.float32(dx) + np.float32(dy) * np.float32(dy)
    listing1 = int(np.float32(np.sqrt(np.float32(f))) + np.float32(0.5))
    assert exact == 40000 and listing1 == 40001
    assert oracle.dist((0, 0), (dx, dy)) == exact


# ----------------------------------------------------------------------------- paper pins

def _read_fig2():
    pts, meta = {}, {}
    with open(os.path.join(GOLDEN, "fig2_worked_example.txt")) as f:
        for line in f:
            line = line.strip()
            if line.startswith("# tour_before") or line.startswith("# tour_after") or line.startswith("# move"):
                k, *v = line[2:].split()
                meta[k] = v
            elif line and not line.startswith("#"):
                c, x, y = line.split()
                pts[c] = (int(x), int(y))
    return pts, meta


def test_fig2_worked_example():
    pts, meta = _read_fig2()
    names = sorted(pts)
    coords = np.array([pts[c] for c in names], dtype=np.int32)
    idx = {c: k for k, c in enumerate(names)}
    before = np.array([idx[c] for c in meta["tour_before"]], dtype=np.int32)
    after = np.array([idx[c] for c in meta["tour_after"]], dtype=np.int32)
    i, j = map(int, meta["move"])
    b, f, d, g = (pts[c] for c in "BFDG")
    # Fig. 2: improving iff distance(b,f) + distance(g,d) > distance(b,d) + distance(g,f)
    fig2_gain = py_dist(b, f) + py_dist(g, d) - py_dist(b, d) - py_dist(g, f)
    assert fig2_gain > 0
    assert oracle.delta(coords, before, i, j) == -fig2_gain
    assert np.array_equal(oracle.apply(before, i, j), after)
    assert oracle.best_move(coords, before) == (i, j, -fig2_gain)
    assert py_length(coords, after) - py_length(coords, before) == -fig2_gain


def test_fig3_cell_numbers():
    with open(os.path.join(GOLDEN, "fig3_cells.txt")) as f:
        rows = [tuple(map(int, l.split())) for l in f if l.strip() and not l.startswith("#")]
    assert len(rows) == 45
    for i, j, printed, reading in rows:
        assert oracle.cell(i, j) == reading
        if j < 9:
            assert printed == reading
    assert sorted(r[3] for r in rows) == list(range(45))


def test_paper_counts():
    vals = {}
    with open(os.path.join(GOLDEN, "paper_counts.txt")) as f:
        for l in f:
            if l.strip() and not l.startswith("#"):
                k, v = l.split()
                vals[k] = int(v)
    assert math.comb(99, 2) == vals["kroE100_swaps"]
    assert math.ceil(math.comb(2392, 2) / (28 * 1024)) == vals["pr2392_iters_28x1024"]
    assert 2048 * 2048 == vals["tile_2048_exchanges"]
    assert 128 * 128 == vals["threads_128x128"]


# ----------------------------------------------------------------------------- brute force

def _small_instances():
    out = []
    for n in (3, 4, 5, 6, 7, 8):
        for seed in (1, 2, 3):
            c = inputs.uniform_coords(n, seed)
            out.append((f"u{n}s{seed}", c, inputs.random_tour(n, seed)))
    for n in (5, 7, 8):
        c = inputs.lattice_coords(n, 4)  # tie-heavy
        out.append((f"lat{n}", c, inputs.random_tour(n, 9)))
    # collinear points and duplicates (d = 0 edges)
    out.append(("line7", np.array([[k * 1000, 5000] for k in (0, 3, 1, 6, 2, 5, 4)], np.int32),
                np.arange(7, dtype=np.int32)))
    out.append(("dup6", np.array([[1, 1], [1, 1], [900, 2], [900, 2], [5, 700], [5, 700]], np.int32),
                np.array([0, 2, 4, 1, 3, 5], np.int32)))
    return out


@pytest.mark.parametrize("name,coords,tour", _small_instances(), ids=lambda v: v if isinstance(v, str) else "")
def test_best_move_brute_force(name, coords, tour):
    nb = brute_neighbours(coords, tour)
    for dl, k, i, j, _ in nb:
        assert oracle.delta(coords, tour, i, j) == dl, (i, j)
    # degenerate pairs always give 0 (reading R1): j = i+1 and (0, n-1)
    n = len(tour)
    for i in range(n - 1):
        assert oracle.delta(coords, tour, i, i + 1) == 0
    assert oracle.delta(coords, tour, 0, n - 1) == 0
    best = min(nb, key=lambda r: (r[0], r[1]))
    assert oracle.best_move(coords, tour) == (best[2], best[3], best[0])


def test_global_optimum_is_2opt_local_minimum():
    for n, seed in ((7, 1), (8, 2), (9, 3)):
        coords = inputs.uniform_coords(n, seed)
        best_len, best_t = None, None
        for perm in itertools.permutations(range(1, n)):
            t = (0,) + perm
            L = py_length(coords, t)
            if best_len is None or L < best_len:
                best_len, best_t = L, t
        bt = np.array(best_t, dtype=np.int32)
        i, j, d = oracle.best_move(coords, bt)
        assert d == 0 and (i, j) == (0, 1)
        res = oracle.local_search(coords, inputs.random_tour(n, seed))
        assert res["status"] == 0 and res["length"] >= best_len
        assert res["length"] == py_length(coords, res["tour"])


def test_vectorised_sweep_matches_on_medium():
    for n, kind in ((60, "uniform"), (120, "lattice"), (257, "uniform")):
        c = inputs.make_coords(kind, n, 5)
        t = inputs.random_tour(n, 6)
        bi, bj, bd, *_ = np_best_move(c, t)
        assert oracle.best_move(c, t) == (bi, bj, bd)


# ----------------------------------------------------------------------------- local search

@pytest.mark.parametrize("kind,n,seed", [("uniform", 100, 1), ("uniform", 100, 2), ("lattice", 100, 1),
                                         ("uniform", 200, 3)])
def test_local_search_trace_invariants(kind, n, seed):
    coords = inputs.make_coords(kind, n, seed)
    tour = inputs.random_tour(n, seed)
    res = oracle.local_search(coords, tour, trace_cap=100_000)
    assert res["status"] == 0
    t = tour.copy()
    L = py_length(coords, t)
    assert len(res["trace"]) == res["iterations"]
    for i, j, d in res["trace"]:
        bi, bj, bd, *_ = np_best_move(coords, t)
        assert (bi, bj, bd) == (i, j, d)          # best move, independent sweep
        assert 0 <= i < j < n and d < 0
        t = np.concatenate([t[: i + 1], t[i + 1 : j + 1][::-1], t[j + 1 :]])
        L2 = py_length(coords, t)
        assert L2 - L == d                        # delta == full recomputation
        L = L2
        assert t[0] == tour[0]
    assert np.array_equal(t, res["tour"])
    assert sorted(t.tolist()) == list(range(n))   # permutation
    assert res["length"] == L
    # local-minimum certificate from the independent vectorised sweep
    _, _, bd, d_all, _, _ = np_best_move(coords, t)
    assert bd == 0 and d_all.min() == 0


def test_convex_position_gives_hull_order():
    n = 64
    ang = np.arange(n) * 2 * np.pi / n
    coords = np.stack([16384 + np.round(15000 * np.cos(ang)), 16384 + np.round(15000 * np.sin(ang))], 1).astype(np.int32)
    tour = inputs.random_tour(n, 3)
    res = oracle.local_search(coords, tour)
    t = res["tour"].tolist()
    k = t.index(0)
    rot = t[k:] + t[:k]
    assert rot == list(range(n)) or rot == [0] + list(range(n - 1, 0, -1))
    hull = sum(py_dist(coords[a], coords[(a + 1) % n]) for a in range(n))
    assert res["length"] == hull


def test_small_n_special_cases():
    c3 = inputs.uniform_coords(3, 1)
    r = oracle.local_search(c3, np.arange(3, dtype=np.int32))
    assert r["iterations"] == 0 and r["status"] == 0
    assert oracle.best_move(c3, np.arange(3, dtype=np.int32)) == (0, 1, 0)
    # n = 4: exactly two structurally non-degenerate pairs, (0,2) and (1,3)
    c4 = np.array([[0, 0], [1000, 1000], [1000, 0], [10, 1300]], np.int32)  # crossing tour
    t4 = np.arange(4, dtype=np.int32)
    nondeg = [(i, j) for j in range(1, 4) for i in range(j) if oracle.delta(c4, t4, i, j) != 0]
    assert nondeg == [(0, 2), (1, 3)]
    r = oracle.local_search(c4, t4)
    assert r["iterations"] == 1 and r["length"] == py_length(c4, [0, 2, 1, 3])


def test_max_iters_status():
    coords = inputs.uniform_coords(100, 1)
    tour = inputs.random_tour(100, 1)
    full = oracle.local_search(coords, tour, trace_cap=10_000)
    capped = oracle.local_search(coords, tour, max_iters=10, trace_cap=100)
    assert capped["status"] == 1 and capped["iterations"] == 10
    assert np.array_equal(capped["trace"], full["trace"][:10])
    zero = oracle.local_search(coords, tour, max_iters=0)
    assert zero["status"] == 1 and zero["iterations"] == 0 and np.array_equal(zero["tour"], tour)
    exact = oracle.local_search(coords, tour, max_iters=full["iterations"])
    assert exact["status"] == 0 and np.array_equal(exact["tour"], full["tour"])
