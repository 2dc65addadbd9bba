"""GPU parity of the batched small-instance local search (SURVEY.md §8(f)
NEXT-3; include/tsp2opt.h tsp2opt_batch_local_search): every instance of the
batch must reach exactly the oracle's local minimum -- same tour, length and
move count -- as if solved alone (oracle.local_search, reading R5 tie-break)."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


def _batch(kind, n, B, seed0, tour="random"):
    cs, ts = [], []
    for b in range(B):
        c = inputs.make_coords(kind, n, seed0 + b)
        cs.append(c)
        ts.append(inputs.make_tour(tour, c, seed0 + b))
    return np.stack(cs).astype(np.int32), np.stack(ts).astype(np.int32)


def _check(cs, ts, out, max_iters=-1):
    for b in range(cs.shape[0]):
        ref = oracle.local_search(cs[b], ts[b], max_iters=max_iters)
        assert out["lengths"][b] == ref["length"], b
        assert out["iterations"][b] == ref["iterations"], b
        assert np.array_equal(out["tours"][b], ref["tour"]), b
        assert out["lengths"][b] == oracle.tour_length(cs[b], out["tours"][b])


@pytest.mark.parametrize("kind,n,B", [("uniform", 100, 64), ("lattice", 100, 32), ("uniform", 3, 5),
                                      ("uniform", 4, 7), ("uniform", 5, 9), ("lattice", 33, 40),
                                      ("uniform", 255, 12), ("uniform", 257, 12), ("lattice", 513, 6),
                                      ("uniform", 1002, 4)])
def test_batch_parity(gpu, kind, n, B):
    cs, ts = _batch(kind, n, B, 11)
    _check(cs, ts, tsp2opt.batch_local_search(cs, ts))


def test_batch_hilbert_and_mixed_starts(gpu):
    cs, ts = _batch("uniform", 200, 10, 5, tour="hilbert")
    ts[::2] = np.stack([inputs.random_tour(200, 100 + b) for b in range(0, 10, 2)])
    _check(cs, ts, tsp2opt.batch_local_search(cs, ts))


@pytest.mark.parametrize("max_iters", [0, 1, 7, 40])
def test_batch_max_iters(gpu, max_iters):
    cs, ts = _batch("uniform", 150, 8, 21)
    _check(cs, ts, tsp2opt.batch_local_search(cs, ts, max_iters=max_iters), max_iters=max_iters)


def test_batch_duplicates_and_collinear(gpu):
    # degenerate geometry: repeated cities (zero edges, many delta ties) and a line
    n = 120
    rng = np.random.default_rng(3)
    dup = rng.integers(0, 6, size=(n, 2)).astype(np.int32) * 5000
    line = np.stack([np.arange(n) * 200, np.full(n, 77)], axis=1).astype(np.int32)
    cs = np.stack([dup, line, inputs.make_coords("lattice", n, 2)])
    ts = np.stack([inputs.random_tour(n, 30 + b) for b in range(3)]).astype(np.int32)
    _check(cs, ts, tsp2opt.batch_local_search(cs, ts))


def test_batch_matches_single_instance_handle(gpu):
    cs, ts = _batch("lattice", 300, 3, 8)
    out = tsp2opt.batch_local_search(cs, ts)
    for b in range(3):
        with tsp2opt.TSP2Opt(cs[b]) as g:
            r = g.local_search(ts[b])
        assert np.array_equal(r["tour"], out["tours"][b]) and r["length"] == out["lengths"][b]


def test_batch_max_n_extreme_coords(gpu):
    # n = 4096 (the shared-memory cap) with coordinates at the range corners
    n = 4096
    c = inputs.make_coords("uniform", n, 9)
    c[:8] = [[0, 0], [32767, 32767], [0, 32767], [32767, 0], [1, 1], [32766, 32766], [0, 1], [32767, 32766]]
    t = inputs.random_tour(n, 9)
    out = tsp2opt.batch_local_search(c[None], t[None], max_iters=60)
    _check(c[None].astype(np.int32), t[None].astype(np.int32), out, max_iters=60)


@pytest.mark.parametrize("packed", ["0", "1"])
@pytest.mark.parametrize("threads", ["32", "96", "256"])
@pytest.mark.parametrize("n", [6, 31, 33, 90, 450])
def test_batch_layouts_and_thread_counts(gpu, monkeypatch, threads, packed, n):
    # both window layouts (packed stream / per-diagonal) for any block size:
    # warp ranges and windows cross diagonals at arbitrary points
    monkeypatch.setenv("TSP2OPT_BATCH_THREADS", threads)
    monkeypatch.setenv("TSP2OPT_BATCH_PACKED", packed)
    cs, ts = _batch("uniform", n, 4, 40 + n)
    _check(cs, ts, tsp2opt.batch_local_search(cs, ts))


def test_batch_async_device_buffers_and_device_validation(gpu):
    import torch
    n, B = 120, 6
    cs, ts = _batch("lattice", n, B, 50)
    bad_t = ts.copy()
    bad_t[2, 5] = bad_t[2, 6]  # not a permutation
    bad_c = cs.copy()
    bad_c[4, 7, 1] = 1 << 15  # out of range
    bad_c[2] = cs[2]
    dc = torch.from_numpy(np.where(np.arange(B)[:, None, None] == 4, bad_c, cs)).cuda()
    dt = torch.from_numpy(bad_t).cuda()
    dl = torch.zeros(B, dtype=torch.int64, device="cuda")
    di = torch.zeros(B, dtype=torch.int64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        tsp2opt.batch_local_search_async(dc.data_ptr(), n, B, dt.data_ptr(), dl.data_ptr(), di.data_ptr(),
                                         stream=s.cuda_stream)
    s.synchronize()
    L, It, T = dl.cpu().numpy(), di.cpu().numpy(), dt.cpu().numpy()
    for b in range(B):
        if b in (2, 4):
            assert L[b] == -1 and It[b] == -1
            assert np.array_equal(T[b], bad_t[b])
            continue
        ref = oracle.local_search(cs[b], ts[b])
        assert (L[b], It[b]) == (ref["length"], ref["iterations"])
        assert np.array_equal(T[b], ref["tour"])
