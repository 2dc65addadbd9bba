"""GPU parity of best-improvement Or-opt (tsp2opt_oropt_*; SURVEY.md §8(f)
NEXT-4 "2.5-opt/Or-opt variants"; L26 §VII; reading R21) against
oracle.*_or -- bit-exact: (i, j, type, delta) per sweep, the traced moves,
final tour, length and move count, through the C ABI."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("n", [3, 4, 5, 6, 7, 16, 33, 100, 481, 1002, 2500])
@pytest.mark.parametrize("kind", ["uniform", "lattice"])
def test_oropt_best_move_parity(gpu, n, kind):
    c = inputs.make_coords(kind, n, 7)
    for t in (inputs.random_tour(n, 7), inputs.random_tour(n, 8), inputs.hilbert_tour(c)):
        assert tsp2opt.oropt_best_move(c, t) == oracle.best_move_or(c, t)


def test_oropt_best_move_c3_sized(gpu):
    n = 7397  # pla7397-shaped: several thousand CTAs of cells and the 2^20-bit key fields
    c = inputs.make_coords("lattice", n, 1)
    for t in (inputs.random_tour(n, 1), inputs.hilbert_tour(c)):
        assert tsp2opt.oropt_best_move(c, t) == oracle.best_move_or(c, t)


@pytest.mark.parametrize("kind,n,seed", [("uniform", 8, 1), ("uniform", 50, 2), ("lattice", 100, 1),
                                         ("uniform", 100, 3), ("lattice", 257, 2), ("uniform", 300, 4)])
def test_oropt_local_search_parity(gpu, kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    t0 = inputs.random_tour(n, seed)
    ref = oracle.local_search_or(c, t0, trace_cap=100_000)
    got = tsp2opt.oropt_local_search(c, t0, trace_cap=100_000)
    assert got["status"] == ref["status"] == 0
    assert got["iterations"] == ref["iterations"]
    assert got["length"] == ref["length"]
    assert np.array_equal(got["tour"], ref["tour"])
    assert np.array_equal(got["trace"].astype(np.int64), ref["trace"])


def test_oropt_duplicates_and_collinear(gpu):
    dup = inputs.make_coords("uniform", 40, 4)
    dup[5] = dup[2]
    dup[17] = dup[2]
    line = np.array([[53 * k % 900, 7] for k in range(41)], dtype=np.int32)
    for c in (dup, line):
        t0 = inputs.random_tour(len(c), 6)
        ref = oracle.local_search_or(c, t0)
        got = tsp2opt.oropt_local_search(c, t0)
        assert (got["length"], got["iterations"]) == (ref["length"], ref["iterations"])
        assert np.array_equal(got["tour"], ref["tour"])


def test_oropt_max_iters(gpu):
    c = inputs.make_coords("uniform", 120, 5)
    t0 = inputs.random_tour(120, 5)
    for cap in (0, 1, 9):
        ref = oracle.local_search_or(c, t0, max_iters=cap)
        got = tsp2opt.oropt_local_search(c, t0, max_iters=cap)
        assert got["status"] == ref["status"] == 1
        assert got["iterations"] == cap and got["length"] == ref["length"]
        assert np.array_equal(got["tour"], ref["tour"])


def test_oropt_local_search_c2_hilbert(gpu):
    # pr1002-shaped from the Hilbert start: full trace parity at a size spanning many CTAs
    n = 1002
    c = inputs.make_coords("uniform", n, 1)
    t0 = inputs.hilbert_tour(c)
    ref = oracle.local_search_or(c, t0, trace_cap=100_000)
    got = tsp2opt.oropt_local_search(c, t0, trace_cap=100_000)
    assert (got["status"], got["iterations"], got["length"]) == (ref["status"], ref["iterations"], ref["length"])
    assert np.array_equal(got["tour"], ref["tour"])
    assert np.array_equal(got["trace"].astype(np.int64), ref["trace"])


@pytest.fixture
def or_mode():
    """Select the Or-opt kernel for one test (tsp2opt_oropt_config), then restore the default."""
    yield tsp2opt.oropt_config
    tsp2opt.oropt_config(-1, 0)


_ORACLE_CACHE = {}


def _oracle_or(kind, n, seed, start):
    key = (kind, n, seed, start)
    if key not in _ORACLE_CACHE:
        c = inputs.make_coords(kind, n, seed)
        t0 = inputs.make_tour(start, c, seed)
        _ORACLE_CACHE[key] = (c, t0, oracle.local_search_or(c, t0, trace_cap=100_000))
    return _ORACLE_CACHE[key]


@pytest.mark.parametrize("filt", [0, 1])
@pytest.mark.parametrize("kind,n,seed,start", [("uniform", 300, 1, "random"), ("lattice", 700, 2, "random"),
                                               ("uniform", 1002, 3, "hilbert"), ("lattice", 1500, 4, "hilbert")])
def test_oropt_local_search_filter_modes(gpu, or_mode, filt, kind, n, seed, start):
    """The whole local search -- every move down to the local minimum, where the deltas
    approach 0 and the FP32 filter's margin matters most -- with the filter forced off
    and on.  Above the n > 2048 default switch: the C3 golden below."""
    or_mode(filt, 0)
    c, t0, ref = _oracle_or(kind, n, seed, start)
    got = tsp2opt.oropt_local_search(c, t0, trace_cap=100_000)
    assert (got["status"], got["iterations"], got["length"]) == (ref["status"], ref["iterations"], ref["length"])
    assert np.array_equal(got["trace"].astype(np.int64), ref["trace"])
    assert np.array_equal(got["tour"], ref["tour"])


def test_oropt_naive_kernel_mode(gpu, or_mode):
    or_mode(-1, 1)
    c = inputs.make_coords("lattice", 400, 9)
    t0 = inputs.random_tour(400, 9)
    ref = oracle.local_search_or(c, t0, trace_cap=100_000)
    got = tsp2opt.oropt_local_search(c, t0, trace_cap=100_000)
    assert np.array_equal(got["trace"].astype(np.int64), ref["trace"]) and np.array_equal(got["tour"], ref["tour"])


def test_oropt_config_errors(gpu):
    for bad in ((-2, 0), (2, 0), (0, 2), (0, -1)):
        with pytest.raises(tsp2opt.TSP2OptError):
            tsp2opt.oropt_config(*bad)


@pytest.mark.parametrize("filt", [-1, 0, 1])
def test_oropt_c3_hilbert_golden(gpu, or_mode, filt):
    """pla7397-shaped C3 from the Hilbert start -- the bench's Or-opt workload -- in the
    default mode (by size: the FP32 filter, n > 2048), the exact walk and the filter
    forced on: every move, the final tour, length and move count equal the committed
    golden (plain oracle, make_golden.py)."""
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "ls_oropt_C3_lattice_hilbert_s1.npz")
    gold = np.load(path)
    or_mode(filt, 0)
    c, _ = inputs.config_instance("C3")
    t0 = inputs.hilbert_tour(c)
    assert np.array_equal(gold["start"], t0)
    k = int(gold["iterations"])
    got = tsp2opt.oropt_local_search(c, t0, trace_cap=k + 10)
    assert (got["status"], got["iterations"], got["length"]) == (0, k, int(gold["length"]))
    assert np.array_equal(got["trace"].astype(np.int64), gold["trace"][:k])
    assert np.array_equal(got["tour"], gold["tour"])
