"""The sharded (NCCL) code path on one GPU: tsp2opt_create_sharded(rank 0,
world 1, id) builds a one-rank communicator, so every sweep runs the 8-byte
ncclAllReduce(MIN) of the packed key on the library's stream exactly as a
multi-GPU rank does (the multi-GPU split itself is covered
by the simulated-shard tests).  Every mode must stay bit-exact with the oracle."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu


def _handle(c):
    return tsp2opt.TSP2Opt(c, 0, 1, tsp2opt.nccl_unique_id())


@pytest.mark.parametrize("kind,n,seed", [("uniform", 1002, 1), ("lattice", 3001, 2)])
def test_nccl_one_rank_local_search(gpu, kind, n, seed):
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    want = oracle.local_search(c, t)
    with _handle(c) as g:
        assert g.best_move(t) == oracle.best_move(c, t)
        res = g.local_search(t)
    assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
    assert np.array_equal(res["tour"], want["tour"])


def test_nccl_one_rank_modes(gpu):
    n = 1500
    c = inputs.make_coords("uniform", n, 3)
    t = inputs.random_tour(n, 3)
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_NEIGHBOURS, 8)  # pruned sweep + allreduce
        res = g.local_search(t)
        want = oracle.pruned_local_search(c, t, 8)
        assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
        g.set_option(tsp2opt.OPT_NEIGHBOURS, 0)
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)  # marker keys reduced, then the exact delta
        res = g.local_search(t, max_iters=500)
        want = oracle.first_local_search(c, t, max_iters=500)
        assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
        assert np.array_equal(res["tour"], want["tour"])
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 0)
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)  # 2.5-opt sweep + allreduce + cooperative apply
        res = g.local_search(t)
        want = oracle.local_search25(c, t)
        assert (res["iterations"], res["length"]) == (want["iterations"], want["length"])
        assert np.array_equal(res["tour"], want["tour"])


def test_nccl_one_rank_full_size_C4(gpu):
    """C4 from the Hilbert start through the NCCL path (incremental culled sweep, the
    allreduce captured in the graph batches): every move equals the oracle's golden."""
    import os
    gold = np.load(os.path.join(os.path.dirname(__file__), "golden", "ls_radius_C4_lattice_hilbert_s1.npz"))
    k = int(gold["iterations"])
    c, t = inputs.config_instance("C4", "hilbert")
    with _handle(c) as g:
        g.set_option(tsp2opt.OPT_TRACE, k + 8)
        res = g.local_search(t)
        trace = g.get_trace(k + 8)
    assert (res["iterations"], res["length"]) == (k, int(gold["length"]))
    assert np.array_equal(np.asarray(trace, np.int64), gold["trace"][:k])
    assert np.array_equal(res["tour"], gold["tour"])
