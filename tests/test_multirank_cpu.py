"""World-size-2 (and 3) CPU coverage of the multi-GPU host logic with gloo.

Each rank takes its shard of the triangular tile space from the library's
host planner (tsp2opt_plan_shard, no GPU), evaluates the oracle over exactly
those tiles, and the ranks combine the packed 64-bit keys with an int64 MIN
allreduce -- the same reduction the product path performs with NCCL.  The
result must equal the unsharded oracle best move on every rank, and the
shards must partition the C(n,2) pairs exactly."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt


def pack(d, i, j):
    return ((d + (1 << 18)) << 44) | (j << 22) | i


def unpack(k):
    return k & 0x3FFFFF, (k >> 22) & 0x3FFFFF, (k >> 44) - (1 << 18)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cases, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    for kind, n, seed in cases:
        c = inputs.make_coords(kind, n, seed)
        t = inputs.random_tour(n, seed)
        plan = tsp2opt.plan_shard(n, rank, world)
        i, j, d = oracle.best_move_tiles(c, t, plan["tiles"], plan["ti"], plan["tj"])
        key = torch.tensor([pack(d, i, j)], dtype=torch.int64)
        dist.all_reduce(key, op=dist.ReduceOp.MIN)
        pairs = torch.tensor([plan["pairs"]], dtype=torch.int64)
        dist.all_reduce(pairs, op=dist.ReduceOp.SUM)
        out.append((unpack(int(key.item())), int(pairs.item())))
    q.put((rank, out))
    dist.destroy_process_group()


CASES = [("uniform", 200, 1), ("lattice", 257, 2), ("uniform", 1002, 3), ("lattice", 613, 4)]


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_min_equals_full(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, CASES, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for idx, (kind, n, seed) in enumerate(CASES):
        c = inputs.make_coords(kind, n, seed)
        t = inputs.random_tour(n, seed)
        want = oracle.best_move(c, t)
        for r in range(world):
            got, pairs = results[r][idx]
            assert got == want
            assert pairs == n * (n - 1) // 2


@pytest.mark.parametrize("n,world", [(100, 2), (1002, 3), (2500, 8), (7397, 8), (33810, 8)])
def test_shards_partition_the_pair_triangle(n, world):
    cover = np.zeros((n, n), dtype=np.int8) if n <= 2500 else None
    total = 0
    for r in range(world):
        plan = tsp2opt.plan_shard(n, r, world)
        total += plan["pairs"]
        if cover is not None:
            for I0, J0 in plan["tiles"]:
                I1, J1 = min(I0 + plan["ti"], n - 1), min(J0 + plan["tj"], n)
                ii, jj = np.meshgrid(np.arange(I0, I1), np.arange(J0, J1), indexing="ij")
                m = ii < jj
                np.add.at(cover, (ii[m], jj[m]), 1)
    assert total == n * (n - 1) // 2
    if cover is not None:
        iu = np.triu_indices(n, 1)
        assert (cover[iu] == 1).all() and cover.sum() == len(iu[0])
    # balance: every shard within one tile of the mean pair count
    loads = [tsp2opt.plan_shard(n, r, world)["pairs"] for r in range(world)]
    p0 = tsp2opt.plan_shard(n, 0, world)
    assert max(loads) - min(loads) <= p0["ti"] * p0["tj"]
