"""GPU parity of the Multiple Fragment (greedy) start tour (SURVEY.md §8(f)
NEXT-1; include/tsp2opt.h tsp2opt_mf_tour; R17, §5.9): the device's
round-parallel construction must give exactly the oracle's sequential greedy
tour, and the local search from it exactly the oracle's local minimum."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


def _mf(c):
    with tsp2opt.TSP2Opt(c) as g:
        return g.mf_tour()


@pytest.mark.parametrize("n", [3, 4, 5, 7, 16, 17, 18, 33, 100, 257, 1002, 2000])
@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_mf_tour_parity(gpu, kind, n):
    for seed in (1, 2):
        c = inputs.make_coords(kind, n, seed)
        r = _mf(c)
        ref = oracle.mf_tour(c)
        assert np.array_equal(r["tour"], ref), (kind, n, seed)
        assert r["length"] == oracle.tour_length(c, ref)
        assert r["rounds"] >= 1


def test_mf_clustered_forces_scans(gpu):
    # 60 tight clusters of 30 cities: every exact 16-nearest list stays inside its
    # cluster, so joining clusters needs the full scans over fragment ends
    rng = np.random.default_rng(7)
    centers = rng.integers(2000, 30000, size=(60, 2))
    c = np.concatenate([ctr + rng.integers(-150, 150, size=(30, 2)) for ctr in centers]).astype(np.int32)
    assert np.array_equal(_mf(c)["tour"], oracle.mf_tour(c))


def test_mf_duplicates_collinear_and_grid(gpu):
    rng = np.random.default_rng(3)
    dup = (rng.integers(0, 8, size=(200, 2)) * 3000).astype(np.int32)  # many zero-length edges and ties
    line = np.stack([rng.permutation(4000)[:300] * 8, np.full(300, 9)], axis=1).astype(np.int32)
    grid = np.array([[x * 500, y * 500] for y in range(20) for x in range(25)], dtype=np.int32)[rng.permutation(500)]
    for c in (dup, line, grid):
        assert np.array_equal(_mf(c)["tour"], oracle.mf_tour(c))


def test_mf_C3_lattice(gpu):
    c, _ = inputs.config_instance("C3")
    assert np.array_equal(_mf(c)["tour"], oracle.mf_tour(c))


def test_mf_then_local_search(gpu):
    for kind, n in (("uniform", 1002), ("lattice", 3000)):
        c = inputs.make_coords(kind, n, 4)
        with tsp2opt.TSP2Opt(c) as g:
            g.mf_tour()
            r = g.local_search_current()
            t, L = g.get_tour()
        ref = oracle.local_search(c, oracle.mf_tour(c))
        assert (r["length"], r["iterations"], L) == (ref["length"], ref["iterations"], ref["length"])
        assert np.array_equal(t, ref["tour"])


def test_mf_repeat_and_reuse_workspace(gpu):
    c = inputs.make_coords("uniform", 500, 9)
    with tsp2opt.TSP2Opt(c) as g:
        a = g.mf_tour()
        g.local_search(inputs.random_tour(500, 1))
        b = g.mf_tour()
    assert np.array_equal(a["tour"], b["tour"]) and a["length"] == b["length"]


def test_mf_full_size_C5_valid(gpu):
    # full size: a permutation starting 0 -> lower-id neighbour, length = recomputed,
    # and (oracle is O(n^2) memory) the greedy edges of a 12000-city prefix instance match
    c, _ = inputs.config_instance("C5")
    r = _mf(c)
    t = r["tour"]
    assert np.array_equal(np.sort(t), np.arange(len(c))) and t[0] == 0 and t[1] < t[-1]
    assert r["length"] == oracle.tour_length(c, t)
    c2 = c[:12000].copy()
    assert np.array_equal(_mf(c2)["tour"], oracle.mf_tour(c2))
