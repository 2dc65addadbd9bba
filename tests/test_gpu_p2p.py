"""The sharded path with the peer-memory exchange (tsp2opt_create_sharded_p2p;
SURVEY §8(a) a6 / §8(e); §VI "dividing the 2-opt task between
multiple devices").

Ranks run as separate PROCESSES (torch.distributed.run, gloo only for the
64-byte mailbox handles) and exchange their shard minima through each other's
mailboxes -- on one GPU the ranks share it (CUDA IPC within one device), on a
multi-GPU box rank r takes GPU r.  Every rank's whole move trace, final tour,
length and iteration count must be identical, and equal to the golden local
search the oracle wrote (tests/golden/, make_golden.py).  A world-1 handle runs
the same kernel in-process.
"""
import hashlib
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))


def _run(world, items, extra=()):
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.join(HERE, "multirank_worker.py"), items,
           "--p2p", *extra]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=1200)
    assert out.returncode == 0, out.stdout[-2000:] + out.stderr[-3000:]
    line = next(x for x in out.stdout.splitlines() if x.startswith("MULTIRANK "))
    return json.loads(line[len("MULTIRANK "):])


def _check_golden(res, variant="radius"):
    for r in res:
        cfg, _, tk = r["item"].partition(":")
        ranks = r["ranks"]
        assert all(x == ranks[0] for x in ranks), ranks
        g = np.load(os.path.join(HERE, "golden", f"ls_{variant}_{cfg}_lattice_{tk}_s1.npz"))
        k = int(g["iterations"])
        r0 = ranks[0]
        assert (r0["iterations"], r0["length"], r0["status"]) == (k, int(g["length"]), 0)
        assert r0["trace"] == hashlib.sha1(g["trace"][:k].astype(np.int64).tobytes()).hexdigest()
        assert r0["tour"] == hashlib.sha1(g["tour"].astype(np.int32).tobytes()).hexdigest()


@pytest.mark.parametrize("world", [2, 3])
def test_p2p_ranks_equal_golden(gpu, world):
    """World 2 and 3 (three shards of unequal tile counts): C3 from the Hilbert and the
    Multiple Fragment starts, every move equal to the oracle's golden trace."""
    _check_golden(_run(world, "C3:hilbert,C3:mf"))


def test_p2p_first_improvement(gpu):
    """First improvement (reading R20): the exchange carries the marker keys, the lowest
    improving cell wins across ranks."""
    _check_golden(_run(2, "C3:mf", ("--first",)), variant="first")


def test_p2p_world1_in_process(gpu):
    c = inputs.uniform_coords(500, 4)
    t = inputs.random_tour(500, 4)
    with tsp2opt.TSP2Opt(c, 0, 1, p2p_allgather=lambda b: [b]) as g:
        assert g.best_move(t) == oracle.best_move(c, t)
        r = g.local_search(t)
    o = oracle.local_search(c, t)
    assert (r["length"], r["iterations"]) == (o["length"], o["iterations"]) and np.array_equal(r["tour"], o["tour"])


def test_p2p_errors(gpu):
    c = inputs.uniform_coords(50, 1)
    h = tsp2opt.create_sharded_p2p(c, 0, 2)
    try:
        with pytest.raises(tsp2opt.TSP2OptError):  # not connected yet
            tsp2opt.best_move(h, inputs.random_tour(50, 1))
        with pytest.raises(tsp2opt.TSP2OptError):  # a world beyond the mailbox width
            tsp2opt.create_sharded_p2p(c, 0, 9)
    finally:
        tsp2opt.destroy(h)
    g = tsp2opt.create(c)
    try:
        with pytest.raises(tsp2opt.TSP2OptError):  # not a p2p handle
            tsp2opt.p2p_export(g)
    finally:
        tsp2opt.destroy(g)


def test_p2p_c4_sharded_incremental(gpu):
    """C4 (571 M pairs) on two ranks: the incremental culled sweep of each rank's half of
    the tile list (the per-shard (row block, column chunk) map, the fused dirty-tile
    kernel, the mailbox exchange between sweep and apply inside the captured graph
    batches) -- every move equals the golden."""
    _check_golden(_run(2, "C4:hilbert"))
