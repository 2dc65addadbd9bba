"""Pins of the exact radius-pruned oracle (oracle_radius_*; SURVEY.md §8(c) "Exact
pruned oracle for large n").  It must return exactly what the plain all-pairs
sweeps return, so every pin compares it against something that does not use
the lemma: explicit brute force over built neighbours, the plain oracle move by
move, the committed C3 golden (written by the plain oracle), and the lemma
itself checked over every improving pair of a vectorised numpy sweep.
"""
import os

import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs
from tests.test_oracle import _small_instances, brute_neighbours, np_best_move
from tests.test_oracle_25opt import _instances as _instances25
from tests.test_oracle_25opt import brute_best25

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.mark.parametrize("name,coords,tour", _small_instances(), ids=lambda v: v if isinstance(v, str) else "")
def test_radius_best_move_brute_force(name, coords, tour):
    """n <= 8, ties, collinear points, duplicate cities: best and first improvement
    equal the explicit neighbour enumeration (L12 Fig. 2 move, reading R5 / R20)."""
    nb = brute_neighbours(coords, tour)
    best = min(nb, key=lambda r: (r[0], r[1]))
    want = (best[2], best[3], best[0]) if best[0] < 0 else (0, 1, 0)
    assert oracle.radius_best_move(coords, tour) == want
    first = next(((i, j, dl) for dl, _, i, j, _ in nb if dl < 0), (0, 1, 0))
    assert oracle.radius_best_move(coords, tour, first=True) == first


@pytest.mark.parametrize("name,coords,tour", _instances25(), ids=lambda v: v if isinstance(v, str) else "")
def test_radius_best_move25_brute_force(name, coords, tour):
    """2.5-opt (reading R19): neighbours built from the move's wording, n <= 12."""
    assert oracle.radius_best_move(coords, tour, node_insertion=True) == brute_best25(coords, tour)


@pytest.mark.parametrize("kind,n,seed", [("uniform", 60, 1), ("lattice", 128, 2), ("uniform", 257, 3),
                                         ("lattice", 500, 4)])
def test_lemma_covers_every_improving_pair(kind, n, seed):
    """Every pair with delta < 0 (vectorised numpy sweep, float64 exact below 2^31)
    has D(i,j) < e_i or D(i+1,j+1) < e_j -- the lemma the pruning rests on."""
    coords = inputs.make_coords(kind, n, seed)
    for tour in (inputs.random_tour(n, seed), inputs.hilbert_tour(coords)):
        _, _, _, d, i, j = np_best_move(coords, tour)
        P = np.asarray(coords, np.int64)[np.r_[tour, tour[:1]]]
        D = lambda a, b: np.floor(np.sqrt(((P[a] - P[b]) ** 2).sum(-1).astype(np.float64)) + 0.5).astype(np.int64)
        e = D(np.arange(n), np.arange(1, n + 1))
        imp = d < 0
        assert imp.any()
        assert np.all((D(i[imp], j[imp]) < e[i[imp]]) | (D(i[imp] + 1, j[imp] + 1) < e[j[imp]]))


@pytest.mark.parametrize("kind", ["uniform", "lattice"])
@pytest.mark.parametrize("n,seed", [(100, 1), (100, 2), (100, 3), (1002, 1), (1002, 2), (1002, 3)])
def test_radius_local_search_equals_plain_move_by_move(kind, n, seed):
    """C1 / C2-shaped (three seeds, uniform and tie-heavy lattice, random start): the
    whole trace -- every move -- final tour, length and iteration count equal the
    plain all-pairs oracle's (L12 §I.B; Table II sizes)."""
    coords = inputs.make_coords(kind, n, seed)
    tour = inputs.random_tour(n, seed)
    a = oracle.local_search(coords, tour, trace_cap=10 * n)
    b = oracle.radius_local_search(coords, tour, trace_cap=10 * n)
    assert a["iterations"] > 0.5 * n
    assert (a["iterations"], a["length"], a["status"]) == (b["iterations"], b["length"], b["status"])
    assert np.array_equal(a["trace"], b["trace"])
    assert np.array_equal(a["tour"], b["tour"])


@pytest.mark.parametrize("kind,n,seed", [("uniform", 100, 1), ("lattice", 150, 2), ("uniform", 240, 3)])
def test_radius_first_and_25opt_equal_plain_move_by_move(kind, n, seed):
    """First improvement (R20) and 2.5-opt (R19): every move equals the plain oracle's."""
    coords = inputs.make_coords(kind, n, seed)
    tour = inputs.random_tour(n, seed)
    a = oracle.first_local_search(coords, tour, trace_cap=100 * n)
    b = oracle.radius_local_search(coords, tour, trace_cap=100 * n, first=True)
    assert a["iterations"] == b["iterations"] and np.array_equal(a["trace"], b["trace"])
    assert np.array_equal(a["tour"], b["tour"]) and a["length"] == b["length"]
    a = oracle.local_search25(coords, tour, trace_cap=100 * n)
    b = oracle.radius_local_search(coords, tour, trace_cap=100 * n, node_insertion=True)
    assert a["iterations"] == b["iterations"] and np.array_equal(a["trace"], b["trace"])
    assert np.array_equal(a["tour"], b["tour"]) and a["length"] == b["length"]
    assert set(np.unique(a["trace"][:, 3])) == {0, 1, 2}


def test_radius_constructive_starts_equal_plain():
    """From Hilbert and Multiple Fragment starts (the C4/C5 golden starts) at n = 1200:
    every move equals the plain oracle's, for all three sweeps."""
    coords = inputs.lattice_coords(1200, 7)
    for tour in (inputs.hilbert_tour(coords), oracle.mf_tour(coords)):
        a = oracle.local_search(coords, tour, trace_cap=5000)
        b = oracle.radius_local_search(coords, tour, trace_cap=5000)
        assert a["iterations"] > 30 and np.array_equal(a["trace"], b["trace"]) and np.array_equal(a["tour"], b["tour"])
        a = oracle.local_search25(coords, tour, trace_cap=5000)
        b = oracle.radius_local_search(coords, tour, trace_cap=5000, node_insertion=True)
        assert np.array_equal(a["trace"], b["trace"]) and np.array_equal(a["tour"], b["tour"])
        a = oracle.first_local_search(coords, tour, trace_cap=20000)
        b = oracle.radius_local_search(coords, tour, trace_cap=20000, first=True)
        assert np.array_equal(a["trace"], b["trace"]) and np.array_equal(a["tour"], b["tour"])


def test_radius_full_size_sweeps_equal_plain():
    """C4 (n = 33810, lattice): the Hilbert start and a tour 40 moves into the search --
    one plain all-pairs sweep of 571 M pairs each -- give the radius sweep's move."""
    coords, _ = inputs.config_instance("C4")
    tour = inputs.hilbert_tour(coords)
    mid = oracle.radius_local_search(coords, tour, max_iters=40)["tour"]
    for t in (tour, mid):
        assert oracle.radius_best_move(coords, t) == oracle.best_move(coords, t)


def test_radius_replays_c3_golden_sampled():
    """The committed C3 golden (plain oracle, 10,050 moves from a random start): the
    golden trace is replayed with oracle.apply, and the radius sweep of the tour before
    move k must give move k for the first 25 moves, every 200th move and the last 25,
    plus (0, 1, 0) at the final tour.  (test_radius_replays_c3_golden_every_move checks
    every move; it takes about 10 minutes on 8 cores, so it runs with TSP2OPT_SLOW=1.)"""
    g = np.load(os.path.join(GOLDEN, "ls_C3_lattice_random_s1.npz"))
    coords, tour = inputs.config_instance("C3")
    tr = g["trace"]
    it = int(g["iterations"])
    ks = set(range(25)) | set(range(0, it, 200)) | set(range(it - 25, it))
    t = tour.copy()
    for k in range(it):
        if k in ks:
            assert oracle.radius_best_move(coords, t) == tuple(int(v) for v in tr[k]), k
        t = oracle.apply(t, int(tr[k, 0]), int(tr[k, 1]))
    assert np.array_equal(t, g["tour"])
    assert oracle.radius_best_move(coords, t) == (0, 1, 0)


@pytest.mark.skipif(os.environ.get("TSP2OPT_SLOW") != "1", reason="about 10 minutes; set TSP2OPT_SLOW=1")
def test_radius_replays_c3_golden_every_move():
    """All 10,050 moves of the committed C3 golden: the radius local search from the same
    random start reproduces the whole trace, the final tour, length and iteration count."""
    g = np.load(os.path.join(GOLDEN, "ls_C3_lattice_random_s1.npz"))
    coords, tour = inputs.config_instance("C3")
    r = oracle.radius_local_search(coords, tour, trace_cap=int(g["iterations"]) + 10)
    assert (r["iterations"], r["length"], r["status"]) == (int(g["iterations"]), int(g["length"]), 0)
    assert np.array_equal(r["trace"], g["trace"][: r["iterations"]])
    assert np.array_equal(r["tour"], g["tour"])


def test_radius_max_iters_status():
    coords = inputs.uniform_coords(200, 5)
    tour = inputs.random_tour(200, 5)
    full = oracle.local_search(coords, tour)
    for cap in (0, 1, 7, full["iterations"]):
        a = oracle.local_search(coords, tour, max_iters=cap)
        b = oracle.radius_local_search(coords, tour, max_iters=cap)
        assert (a["status"], a["iterations"], a["length"]) == (b["status"], b["iterations"], b["length"])
        assert np.array_equal(a["tour"], b["tour"])
