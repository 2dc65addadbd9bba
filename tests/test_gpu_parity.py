"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Integer work throughout (exact EUC_2D nint distances, integer deltas, indices),
so the bar is equality of (i, j, delta) per sweep, final tour, length and
iteration count (north_star)."""
import os

import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _inst(kind, n, seed, tour="random"):
    c = inputs.make_coords(kind, n, seed)
    return c, inputs.make_tour(tour, c, seed)


def test_selftest_exhaustive_distance_and_filter(gpu):
    r = tsp2opt.selftest()
    assert r["dist_violations"] == 0, f"exact nint(sqrt(s)) wrong for some s in [0, 2*32767^2]: {r}"
    assert r["filter_violations"] == 0, f"squared-distance prefilter rejects a reachable (dx, dy): {r}"


def test_selftest_sqrt_error_bound(gpu):
    """The sqrt-sum prefilter's 0.5 slack needs a relative MUFU.SQRT
    error <= 2^-21 on every float the filter can see."""
    r = tsp2opt.selftest_sqrt()
    assert r["zero_ok"]
    assert 0 <= r["max_rel_err"] <= 2.0 ** -21, r


SIZES = [3, 4, 5, 7, 16, 31, 32, 33, 100, 101, 479, 480, 481, 961, 1002, 1921, 2500]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_best_move_parity_sizes(gpu, n, kind):
    c, t = _inst(kind, n, 3)
    with tsp2opt.TSP2Opt(c) as g:
        for seed in (3, 4):
            t = inputs.random_tour(n, seed)
            assert g.best_move(t) == oracle.best_move(c, t)
        # hilbert start: short edges, mostly filtered pairs
        th = inputs.hilbert_tour(c)
        assert g.best_move(th) == oracle.best_move(c, th)


@pytest.mark.parametrize("bounds", ["0", "1", "2", "3"])
@pytest.mark.parametrize("rows", [7, 15])
@pytest.mark.parametrize("warps,tj", [(1, 2), (1, 3), (1, 32), (2, 64), (4, 128), (4, 1024), (3, 7)])
def test_best_move_parity_geometries(gpu, monkeypatch, rows, warps, tj, bounds):
    # tiny and odd tiles exercise masked diagonal tiles and ragged column tails,
    # for both instantiated row counts R, with and without tile-level bounds
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    monkeypatch.setenv("TSP2OPT_ROWS", str(rows))
    monkeypatch.setenv("TSP2OPT_WARPS", str(warps))
    monkeypatch.setenv("TSP2OPT_TJ", str(tj))
    for kind, n in (("uniform", 1002), ("lattice", 2000), ("uniform", 97)):
        c, t = _inst(kind, n, 5)
        with tsp2opt.TSP2Opt(c) as g:
            geo = g.geometry()
            assert (geo["rows"], geo["warps"], geo["tj"]) == (rows, warps, tj)
            assert geo["pairs"] == n * (n - 1) // 2
            assert g.best_move(t) == oracle.best_move(c, t)


@pytest.mark.parametrize("kind,n,seed", [("uniform", 100, 1), ("uniform", 100, 2), ("uniform", 100, 3),
                                         ("lattice", 100, 1)])
def test_trace_parity_C1(gpu, kind, n, seed):
    """Every sweep of the local search: best move, then the explicit apply."""
    c, t = _inst(kind, n, seed)
    ref = oracle.local_search(c, t, trace_cap=10_000)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_tour(t)
        for i, j, d in ref["trace"]:
            assert g.best_move() == (i, j, d)
            g.apply(i, j)
        assert g.best_move() == (0, 1, 0)
        tour, L = g.get_tour()
        assert np.array_equal(tour, ref["tour"]) and L == ref["length"]


@pytest.mark.parametrize("kind,n,seed", [("uniform", 100, 1), ("lattice", 100, 1), ("uniform", 1002, 1),
                                         ("uniform", 1002, 2), ("uniform", 1002, 3), ("lattice", 1002, 1),
                                         ("lattice", 1002, 2), ("uniform", 2000, 7)])
def test_local_search_parity(gpu, kind, n, seed):
    c, t = _inst(kind, n, seed)
    ref = oracle.local_search(c, t)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_TILE_BOUNDS, seed % 4)  # every filter form over the seeds
        res = g.local_search(t)
        assert res["status"] == tsp2opt.OK
        assert res["iterations"] == ref["iterations"]
        assert res["length"] == ref["length"] == oracle.tour_length(c, res["tour"])
        assert np.array_equal(res["tour"], ref["tour"])
        # determinism: a second run is bit-identical
        res2 = g.local_search(t)
        assert np.array_equal(res2["tour"], res["tour"]) and res2["iterations"] == res["iterations"]


def test_local_search_parity_C3_golden(gpu):
    path = os.path.join(GOLDEN, "ls_C3_lattice_random_s1.npz")
    if not os.path.exists(path):
        pytest.fail("golden file missing: run tests/golden/make_golden.py C3")
    gold = np.load(path)
    c, t = inputs.config_instance("C3")
    with tsp2opt.TSP2Opt(c) as g:
        res = g.local_search(t)
        assert res["iterations"] == int(gold["iterations"])
        assert res["length"] == int(gold["length"])
        assert np.array_equal(res["tour"], gold["tour"])
        # the first moves of the trace, sweep by sweep
        g.set_tour(t)
        for i, j, d in gold["trace"][:50]:
            assert g.best_move() == (int(i), int(j), int(d))
            g.apply(int(i), int(j))


def test_max_iters_parity(gpu):
    c, t = _inst("uniform", 1002, 2)
    with tsp2opt.TSP2Opt(c) as g:
        for cap in (0, 1, 7, 100):
            ref = oracle.local_search(c, t, max_iters=cap)
            res = g.local_search(t, max_iters=cap)
            assert res["status"] == ref["status"] and res["iterations"] == ref["iterations"]
            assert res["length"] == ref["length"] and np.array_equal(res["tour"], ref["tour"])


@pytest.mark.parametrize("bounds", ["1", "2", "3"])
@pytest.mark.parametrize("world", [2, 3, 8])
def test_simulated_shards_min_equals_full(gpu, monkeypatch, world, bounds):
    """Every shard's sweep, then the min over shards == the unsharded sweep ==
    the oracle; with the culled sweep (bounds 2) the tours are spatially
    coherent (Hilbert order) so most tiles of every shard are culled."""
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)
    for kind, n in (("uniform", 1002), ("lattice", 7397)):
        c, t = _inst(kind, n, 2, "hilbert" if bounds in ("2", "3") else "random")
        with tsp2opt.TSP2Opt(c) as g:
            full = g.best_move(t)
            keys, pairs = [], 0
            for r in range(world):
                g.debug_set_shard(r, world)
                pairs += g.geometry()["pairs"]
                i, j, d = g.best_move()
                keys.append((d, j * (j - 1) // 2 + i, i, j))
            g.debug_set_shard(0, 1)
            assert pairs == n * (n - 1) // 2
            d, _, i, j = min(keys)
            assert (i, j, d) == full == oracle.best_move(c, t)


def test_apply_explicit_matches_oracle(gpu):
    c, t = _inst("uniform", 501, 4)
    rng = np.random.default_rng(0)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_tour(t)
        ref = t.copy()
        for _ in range(40):
            i, j = sorted(rng.choice(501, 2, replace=False).tolist())
            g.apply(i, j)
            ref = oracle.apply(ref, i, j)
        for i, j in ((0, 1), (0, 500), (499, 500), (0, 2), (1, 500)):
            g.apply(i, j)
            ref = oracle.apply(ref, i, j)
        tour, L = g.get_tour()
        assert np.array_equal(tour, ref) and L == oracle.tour_length(c, ref)
        assert g.best_move() == oracle.best_move(c, ref)


def test_errors_and_no_state_change(gpu):
    c, t = _inst("uniform", 50, 1)
    with tsp2opt.TSP2Opt(c) as g:
        with pytest.raises(tsp2opt.TSP2OptError) as e:
            g.best_move()
        assert e.value.code == tsp2opt.ESTATE
        g.set_tour(t)
        before = g.get_tour()
        bad = t.copy()
        bad[3] = bad[4]
        for tour, code in ((bad, tsp2opt.ENOTPERM), (np.r_[t[:-1], 50].astype(np.int32), tsp2opt.ENOTPERM)):
            with pytest.raises(tsp2opt.TSP2OptError) as e:
                g.set_tour(tour)
            assert e.value.code == code
        for i, j in ((3, 3), (5, 2), (-1, 4), (0, 50)):
            with pytest.raises(tsp2opt.TSP2OptError) as e:
                g.apply(i, j)
            assert e.value.code == tsp2opt.EINVAL
        after = g.get_tour()
        assert np.array_equal(before[0], after[0]) and before[1] == after[1]
        assert g.best_move() == oracle.best_move(c, t)


def test_device_tour_path(gpu):
    import torch
    c, t = _inst("lattice", 3000, 2)
    with tsp2opt.TSP2Opt(c) as g:
        dt = torch.from_numpy(t).cuda()
        g.set_stream(torch.cuda.current_stream().cuda_stream)
        g.set_tour_device_async(dt.data_ptr())
        g.iterate_async(3)
        s = g.sync()
        ref = oracle.local_search(c, t, max_iters=3, trace_cap=3)
        assert s["iterations"] == 3 and s["length"] == ref["length"]
        assert g.get_tour()[0].tolist() == ref["tour"].tolist()
        bad = dt.clone()
        bad[10] = bad[11]
        g.set_tour_device_async(bad.data_ptr())
        with pytest.raises(tsp2opt.TSP2OptError) as e:
            g.sync()
        assert e.value.code == tsp2opt.ENOTPERM
        g.set_stream(None)


def test_small_n_cases(gpu):
    c3 = inputs.uniform_coords(3, 1)
    with tsp2opt.TSP2Opt(c3) as g:
        r = g.local_search(np.arange(3, dtype=np.int32))
        assert r["iterations"] == 0 and r["status"] == 0
        assert g.best_move() == (0, 1, 0)
    dup = np.array([[1, 1], [1, 1], [900, 2], [900, 2], [5, 700], [5, 700]], np.int32)
    t = np.array([0, 2, 4, 1, 3, 5], np.int32)
    with tsp2opt.TSP2Opt(dup) as g:
        res = g.local_search(t)
        ref = oracle.local_search(dup, t)
        assert np.array_equal(res["tour"], ref["tour"]) and res["length"] == ref["length"]


@pytest.mark.parametrize("persistent", ["0", "1"])
@pytest.mark.parametrize("kind,n,seed", [("uniform", 1002, 5), ("lattice", 3001, 6), ("uniform", 97, 7),
                                         ("lattice", 2000, 8)])
def test_local_search_parity_both_loops(gpu, monkeypatch, persistent, kind, n, seed):
    """The persistent single-launch loop and the per-iteration kernel loop (used by
    sharded handles) reach the oracle's local minimum identically, with and
    without per-tile seeding."""
    monkeypatch.setenv("TSP2OPT_PERSISTENT", persistent)
    monkeypatch.setenv("TSP2OPT_SEED", "1" if seed % 2 else "0")
    c, t = _inst(kind, n, seed)
    ref = oracle.local_search(c, t)
    with tsp2opt.TSP2Opt(c) as g:
        res = g.local_search(t)
        assert (res["iterations"], res["length"]) == (ref["iterations"], ref["length"])
        assert np.array_equal(res["tour"], ref["tour"])
        capped = g.local_search(t, max_iters=17)
        want = oracle.local_search(c, t, max_iters=17)
        assert capped["status"] == want["status"] and np.array_equal(capped["tour"], want["tour"])


@pytest.mark.parametrize("bounds", ["1", "2", "3"])
@pytest.mark.parametrize("rows", [7, 15])
def test_seeded_sweeps_mixed_operations(gpu, monkeypatch, rows, bounds):
    """Each sweep after a device-resident move is seeded with the previous sweep's
    surviving tile minima; interleave every operation that could make those
    stale (best_move sweeps, explicit applies, new tours, shard changes) and
    check each following sweep against the oracle."""
    monkeypatch.setenv("TSP2OPT_ROWS", str(rows))
    monkeypatch.setenv("TSP2OPT_SEED", "1")
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", bounds)  # 2: culled tiles must reset their seeds
    monkeypatch.setenv("TSP2OPT_CULL_ROWS", str(rows))  # 3: stored tile minima across every state change
    c, t = _inst("lattice", 3001, 8)
    rng = np.random.default_rng(3)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_tour(t)

        def check():
            tour, L = g.get_tour()
            assert L == oracle.tour_length(c, tour)
            assert g.best_move() == oracle.best_move(c, tour)

        for rnd in range(6):
            g.iterate_async(int(rng.integers(1, 5)))
            g.sync()
            check()                       # best_move right after seeded iterations
            g.iterate_async(2)            # ... and iterations right after a best_move sweep
            g.sync()
            check()
            i, j = sorted(rng.choice(3001, 2, replace=False).tolist())
            g.apply(i, j)                 # explicit (non-improving) move
            g.iterate_async(1)
            g.sync()
            check()
            if rnd == 3:
                g.debug_set_shard(1, 3)   # a different tile list
                g.debug_set_shard(0, 1)
                g.iterate_async(2)
                g.sync()
                check()
            if rnd == 4:
                g.set_tour(inputs.random_tour(3001, 99))
                g.iterate_async(3)
                g.sync()
                check()


@pytest.mark.parametrize("kind,n,iters,seed", [("uniform", 8, 20, 1), ("uniform", 100, 60, 2), ("lattice", 100, 40, 3),
                                               ("uniform", 200, 30, 4), ("uniform", 1002, 8, 5), ("lattice", 1002, 8, 6)])
def test_ils_parity(gpu, kind, n, iters, seed):
    """Iterated Local Search (L10 Algorithm 1, double-bridge perturbation):
    the best length after every step, the final tour and length match the oracle."""
    c, t = _inst(kind, n, seed)
    ref = oracle.ils(c, t, iters, seed=1000 + seed)
    with tsp2opt.TSP2Opt(c) as g:
        res = g.ils(t, iters, 1000 + seed)
        assert res["lengths"].tolist() == ref["lengths"].tolist()
        assert res["length"] == ref["length"] and np.array_equal(res["tour"], ref["tour"])
        tour, L = g.get_tour()  # the handle holds the best tour afterwards
        assert np.array_equal(tour, ref["tour"]) and L == ref["length"]


@pytest.mark.parametrize("cull_tj", ["2", "3", "32", "64"])
@pytest.mark.parametrize("rows", [7, 15])
@pytest.mark.parametrize("kind,n,seed,start", [("uniform", 2000, 11, "random"), ("lattice", 3001, 12, "hilbert")])
def test_incremental_culled_local_search(gpu, monkeypatch, cull_tj, rows, kind, n, seed, start):
    """TSP2OPT_OPT_TILE_BOUNDS = 3: after each move only the tiles with a row or
    column position in the move's [i, j] are culled / re-swept and the others
    keep their stored minimum; the whole move trace must equal the oracle's."""
    monkeypatch.setenv("TSP2OPT_TILE_BOUNDS", "3")
    monkeypatch.setenv("TSP2OPT_CULL_TJ", cull_tj)
    monkeypatch.setenv("TSP2OPT_CULL_ROWS", str(rows))
    c, t = _inst(kind, n, seed, start)
    ref = oracle.local_search(c, t, trace_cap=10 * n)
    with tsp2opt.TSP2Opt(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, 10 * n)
        res = g.local_search(t)
        trace = g.get_trace(10 * n)
    assert (res["iterations"], res["length"]) == (ref["iterations"], ref["length"])
    assert np.array_equal(res["tour"], ref["tour"])
    assert np.array_equal(np.asarray(trace, dtype=np.int64), ref["trace"])
