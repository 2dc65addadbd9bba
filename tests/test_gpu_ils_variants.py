"""Iterated Local Search (L10 Algorithm 1) over every local-search variant of the
handle: pruned (R18), first improvement (R20), pruned + first, 2.5-opt (R19);
bit-exact with oracle.ils(..., variant) -- best length after every step and the
final tour."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu

VARIANTS = [dict(neighbours=8), dict(first=True), dict(neighbours=6, first=True), dict(node_insertion=True)]


@pytest.mark.parametrize("kw", VARIANTS, ids=["pruned8", "first", "pruned6-first", "2.5opt"])
@pytest.mark.parametrize("kind,n,iters,seed", [("uniform", 100, 20, 1), ("lattice", 200, 10, 2), ("uniform", 400, 3, 3)])
def test_ils_variant_parity(gpu, kw, kind, n, iters, seed):
    c = inputs.make_coords(kind, n, seed)
    t = inputs.random_tour(n, seed)
    want = oracle.ils(c, t, iters, 2013 + seed, **kw)
    with tsp2opt.TSP2Opt(c) as g:
        if kw.get("neighbours"):
            g.set_option(tsp2opt.OPT_NEIGHBOURS, kw["neighbours"])
        if kw.get("first"):
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
        if kw.get("node_insertion"):
            g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
        got = g.ils(t, iters, 2013 + seed)
    assert got["lengths"].tolist() == want["lengths"].tolist()
    assert got["length"] == want["length"] and np.array_equal(got["tour"], want["tour"])
