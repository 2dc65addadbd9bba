"""GPU parity of the batched Iterated Local Search (L10 Algorithm 1; SURVEY.md
§8(f) NEXT-2 "batched multi-replica runs for n < 200"; include/tsp2opt.h
tsp2opt_batch_ils): every replica must follow oracle.ils step by step -- the
best length after every ILS step, the final tour and length (readings R14-R16:
same double-bridge cuts from the replica's seed, strict-improvement acceptance)."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


def _batch(kind, n, B, seed0):
    cs, ts = [], []
    for b in range(B):
        c = inputs.make_coords(kind, n, seed0 + b)
        cs.append(c)
        ts.append(inputs.make_tour("random", c, seed0 + b))
    return np.stack(cs).astype(np.int32), np.stack(ts).astype(np.int32)


def _check(cs, ts, iters, seeds, out):
    for b in range(cs.shape[0]):
        ref = oracle.ils(cs[b], ts[b], iters, int(seeds[b]))
        assert out["history"][b].tolist() == ref["lengths"].tolist(), b
        assert out["lengths"][b] == ref["length"], b
        assert np.array_equal(out["tours"][b], ref["tour"]), b
        assert out["lengths"][b] == oracle.tour_length(cs[b], out["tours"][b])


@pytest.mark.parametrize("kind,n,B,iters", [("uniform", 100, 16, 30), ("lattice", 100, 8, 30), ("uniform", 8, 6, 20),
                                            ("uniform", 7, 4, 5), ("uniform", 3, 3, 4), ("uniform", 200, 6, 12),
                                            ("lattice", 257, 3, 6), ("uniform", 513, 2, 4)])
def test_batch_ils_parity(gpu, kind, n, B, iters):
    cs, ts = _batch(kind, n, B, 70)
    seeds = np.arange(B, dtype=np.uint64) * np.uint64(7919) + np.uint64(2013)
    _check(cs, ts, iters, seeds, tsp2opt.batch_ils(cs, ts, iters, seeds))


def test_batch_ils_multistart_one_instance(gpu):
    """Multi-start on ONE instance (the paper's ILS setting): replicas share the
    coordinates and differ in start tour and seed; the best replica is the
    minimum of the oracle's runs."""
    n, B, iters = 100, 12, 25
    c = inputs.make_coords("uniform", n, 5).astype(np.int32)
    cs = np.repeat(c[None], B, axis=0)
    ts = np.stack([inputs.make_tour("random", c, 100 + b) for b in range(B)]).astype(np.int32)
    seeds = np.array([2 ** 63 + 12345 * b for b in range(B)], dtype=np.uint64)  # high bit set: uint64 path
    out = tsp2opt.batch_ils(cs, ts, iters, seeds)
    _check(cs, ts, iters, seeds, out)
    assert out["lengths"].min() == min(oracle.ils(c, ts[b], iters, int(seeds[b]))["length"] for b in range(B))


def test_batch_ils_matches_handle_ils(gpu):
    c = inputs.make_coords("lattice", 150, 3).astype(np.int32)
    t = inputs.make_tour("random", c, 3).astype(np.int32)
    out = tsp2opt.batch_ils(c[None], t[None], 15, [99])
    with tsp2opt.TSP2Opt(c) as g:
        res = g.ils(t, 15, 99)
    assert out["history"][0].tolist() == res["lengths"].tolist()
    assert np.array_equal(out["tours"][0], res["tour"]) and out["lengths"][0] == res["length"]


def test_batch_ils_zero_iterations_is_local_search(gpu):
    cs, ts = _batch("uniform", 90, 5, 3)
    out = tsp2opt.batch_ils(cs, ts, 0, np.zeros(5, dtype=np.uint64))
    ls = tsp2opt.batch_local_search(cs, ts)
    assert np.array_equal(out["tours"], ls["tours"]) and np.array_equal(out["lengths"], ls["lengths"])
    assert np.array_equal(out["history"][:, 0], ls["lengths"])


def test_batch_ils_async_device_validation(gpu):
    import torch
    n, B, iters = 64, 4, 6
    cs, ts = _batch("lattice", n, B, 9)
    bad_t = ts.copy()
    bad_t[1, 3] = bad_t[1, 4]  # not a permutation
    seeds = np.arange(B, dtype=np.uint64) + np.uint64(5)
    dc = torch.from_numpy(cs).cuda()
    dt = torch.from_numpy(bad_t).cuda()
    ds = torch.from_numpy(seeds.view(np.int64)).cuda()
    dl = torch.zeros(B, dtype=torch.int64, device="cuda")
    dh = torch.zeros(B, iters + 1, dtype=torch.int64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        tsp2opt.batch_ils_async(dc.data_ptr(), n, B, dt.data_ptr(), iters, ds.data_ptr(), dl.data_ptr(),
                                dh.data_ptr(), stream=s.cuda_stream)
    s.synchronize()
    L, T, H = dl.cpu().numpy(), dt.cpu().numpy(), dh.cpu().numpy()
    for b in range(B):
        if b == 1:
            assert L[b] == -1 and np.array_equal(T[b], bad_t[b])
            continue
        ref = oracle.ils(cs[b], ts[b], iters, int(seeds[b]))
        assert H[b].tolist() == ref["lengths"].tolist() and L[b] == ref["length"]
        assert np.array_equal(T[b], ref["tour"])


def test_batch_ils_errors(gpu):
    cs, ts = _batch("uniform", 20, 2, 1)
    with pytest.raises(tsp2opt.TSP2OptError):
        tsp2opt.batch_ils(cs, ts, -1, [1, 2])
    bad = ts.copy()
    bad[0, 0] = bad[0, 1]
    with pytest.raises(tsp2opt.TSP2OptError):
        tsp2opt.batch_ils(cs, bad, 3, [1, 2])
