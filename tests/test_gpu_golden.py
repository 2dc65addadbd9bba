"""Every move of the full local searches at BASELINE.json's sizes equals the oracle's.

The golden files under tests/golden/ were written by tests/golden/make_golden.py,
which calls only oracle/: the exact radius-pruned oracle (identical to the plain
all-pairs oracle by the lemma of SURVEY.md §8(c); pinned move by move in
tests/test_oracle_radius.py) for best-improvement 2-opt, first improvement
(reading R20) and 2.5-opt (R19), oracle.pruned_local_search for the K = 8
neighbourhood (R18), and the plain oracle's Multiple Fragment tour (R17) as the
`mf` start.  Each test runs the library in its default launch configuration
(the one bench.py times) with the move trace on, and compares the WHOLE trace
(i, j, delta[, type]) move by move, the final tour, length, iteration count and
status -- the north_star bar "bit-exact ... in best move per sweep, final tour,
final length and iteration count" (§I.B local minimum; L22 Table II
sizes pla7397 / pla33810 / pla85900).
"""
import glob
import os

import numpy as np
import pytest

from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _goldens():
    out = []
    for p in sorted(glob.glob(os.path.join(GOLDEN, "ls_*_C[345]_lattice_*_s1.npz"))):
        name = os.path.basename(p)[3:-4]
        parts = name.split("_")
        if len(parts) != 5:  # ls_C3_lattice_random_s1.npz (round 1, plain oracle): test_gpu_parity.py
            continue
        variant, cfg, _, tk, _ = parts
        if variant == "oropt":  # the stateless Or-opt path: tests/test_gpu_oropt.py
            continue
        out.append(pytest.param(variant, cfg, tk, p, id=f"{variant}-{cfg}-{tk}"))
    return out


def _options(g, variant):
    if variant == "first":
        g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
    elif variant == "25opt":
        g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
    elif variant.startswith("knn"):
        g.set_option(tsp2opt.OPT_NEIGHBOURS, int(variant[3:]))
    else:
        assert variant == "radius", variant


@pytest.mark.parametrize("variant,cfg,tk,path", _goldens())
def test_full_local_search_every_move(gpu, variant, cfg, tk, path):
    gold = np.load(path)
    coords, _ = inputs.config_instance(cfg)
    start = gold["start"]
    k = int(gold["iterations"])
    typed = variant == "25opt"
    with tsp2opt.TSP2Opt(coords) as g:
        if tk == "mf":
            # the device Multiple Fragment tour equals the oracle's (reading R17), then the
            # search continues on the device from it (Table II protocol, L22 §V)
            m = g.mf_tour()
            assert np.array_equal(m["tour"], start)
        else:
            assert np.array_equal(start, inputs.make_tour(tk, coords, 1))
        _options(g, variant)
        g.set_option(tsp2opt.OPT_TRACE, k + 16)
        res = g.local_search_current() if tk == "mf" else g.local_search(start)
        if tk == "mf":
            res["tour"] = g.get_tour()[0]
        trace = g.get_trace_typed(k + 16) if typed else g.get_trace(k + 16)
    assert (res["iterations"], res["length"], res["status"]) == (k, int(gold["length"]), int(gold["status"]))
    assert len(trace) == k
    want = gold["trace"][:k]
    got = np.asarray(trace, dtype=np.int64)
    bad = np.nonzero((got != want).any(axis=1))[0]
    assert bad.size == 0, f"first differing move {bad[:1]}: got {got[bad[:1]]}, want {want[bad[:1]]}"
    assert np.array_equal(res["tour"], gold["tour"])


def test_goldens_present():
    """The C4 / C5 goldens of every variant the GPU path offers at those sizes exist."""
    have = {(p.values[0], p.values[1], p.values[2]) for p in _goldens()}
    for cfg in ("C4", "C5"):
        assert ("radius", cfg, "hilbert") in have
        for v in ("radius", "first", "25opt", "knn8"):
            assert (v, cfg, "mf") in have, (v, cfg)
