"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This module holds NO arithmetic of the 2-opt method (no distances, no deltas,
no moves): only counter-based random numbers and the instance / start-tour
recipes of DESIGN.md "Input recipe".  Both sides receive the
same int32 arrays from here; neither side imports the other.

Recipes (all driven by splitmix64, Steele et al.):
  * uniform   -- x = next() >> 49, y = next() >> 49 (15-bit integer coords), the
                 TSPLIB kroA100/pr1002-shaped instances (Table II
                 rows; the paper's instances are TSPLIB files).
  * lattice   -- "pla"-shaped VLSI-like instances: n distinct sites of a G x G
                 grid, G = ceil(sqrt(2n)), pitch floor(32767 / G), chosen by a
                 partial Fisher-Yates shuffle; tie-heavy (many equal distances).
  * random tour  -- Fisher-Yates, r = next() % (k+1) for k = n-1 .. 1
                 (§V "the initial solution s0 is a random tour").
  * hilbert tour -- cities sorted by (Hilbert index on the 2^15 grid, city id),
                 a deterministic constructive start standing in for the paper's
                 Multiple-Fragment start (§V; reading R9).
"""
from __future__ import annotations

import math

import numpy as np

_GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

COORD_BITS = 15
COORD_LIMIT = 1 << COORD_BITS  # coordinates are integers in [0, 2^15)


def splitmix64(seed: int, count: int, offset: int = 0) -> np.ndarray:
    """Outputs offset..offset+count-1 of the splitmix64 stream seeded with `seed`.

    Output k is mix(seed + (k+1)*gamma), so the stream is counter-based and can
    be produced vectorised (and identically in C, see tests/test_inputs.py).
    """
    with np.errstate(over="ignore"):
        k = np.arange(offset + 1, offset + count + 1, dtype=np.uint64)
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + k * _GAMMA
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_coords(n: int, seed: int) -> np.ndarray:
    """int32[n, 2] uniform integer coordinates in [0, 2^15)."""
    r = splitmix64(seed, 2 * n) >> np.uint64(64 - COORD_BITS)
    return r.astype(np.int32).reshape(n, 2)


def lattice_coords(n: int, seed: int) -> np.ndarray:
    """int32[n, 2]: n distinct sites of a G x G lattice (pla-shaped, tie-heavy)."""
    g = math.isqrt(2 * n)
    if g * g < 2 * n:
        g += 1
    pitch = (COORD_LIMIT - 1) // g
    sites = np.arange(g * g, dtype=np.int64)
    total = g * g
    rnd = splitmix64(seed ^ 0x5A5A5A5A, n)
    # partial Fisher-Yates: position k receives a uniformly chosen remaining site
    for k in range(n):
        r = k + int(rnd[k] % np.uint64(total - k))
        sites[k], sites[r] = sites[r], sites[k]
    chosen = sites[:n]
    xy = np.empty((n, 2), dtype=np.int32)
    xy[:, 0] = (chosen % g) * pitch
    xy[:, 1] = (chosen // g) * pitch
    return xy


def make_coords(kind: str, n: int, seed: int) -> np.ndarray:
    if kind == "uniform":
        return uniform_coords(n, seed)
    if kind == "lattice":
        return lattice_coords(n, seed)
    raise ValueError(f"unknown instance kind {kind!r}")


def random_tour(n: int, seed: int) -> np.ndarray:
    """int32[n] uniformly random permutation (Fisher-Yates, k = n-1 .. 1)."""
    t = np.arange(n, dtype=np.int64)
    rnd = splitmix64(seed ^ 0x7A7A7A7A7A7A7A7A, max(n - 1, 0))
    for idx, k in enumerate(range(n - 1, 0, -1)):
        r = int(rnd[idx] % np.uint64(k + 1))
        t[k], t[r] = t[r], t[k]
    return t.astype(np.int32)


def hilbert_index(x: np.ndarray, y: np.ndarray, order: int = COORD_BITS) -> np.ndarray:
    """Hilbert-curve index of integer points on the 2^order grid (vectorised xy2d)."""
    x = x.astype(np.int64).copy()
    y = y.astype(np.int64).copy()
    d = np.zeros_like(x)
    s = 1 << (order - 1)
    while s > 0:
        rx = ((x & s) > 0).astype(np.int64)
        ry = ((y & s) > 0).astype(np.int64)
        d += s * s * ((3 * rx) ^ ry)
        # rotate the quadrant
        flip = ry == 0
        swap_mask = flip & (rx == 1)
        x = np.where(swap_mask, s - 1 - x, x)
        y = np.where(swap_mask, s - 1 - y, y)
        xs = np.where(flip, y, x)
        ys = np.where(flip, x, y)
        x, y = xs, ys
        s >>= 1
    return d


def hilbert_tour(coords: np.ndarray) -> np.ndarray:
    """int32[n]: cities ordered by (Hilbert index, city id)."""
    h = hilbert_index(coords[:, 0], coords[:, 1])
    ids = np.arange(coords.shape[0], dtype=np.int64)
    return np.lexsort((ids, h)).astype(np.int32)


def make_tour(kind: str, coords: np.ndarray, seed: int) -> np.ndarray:
    if kind == "random":
        return random_tour(coords.shape[0], seed)
    if kind == "hilbert":
        return hilbert_tour(coords)
    if kind == "identity":
        return np.arange(coords.shape[0], dtype=np.int32)
    raise ValueError(f"unknown tour kind {kind!r}")


# The workloads named by BASELINE.json `configs`.
CONFIGS = {
    "C1": dict(n=100, coords="uniform", seed=1, tour="random"),
    "C2": dict(n=1002, coords="uniform", seed=1, tour="random"),
    "C3": dict(n=7397, coords="lattice", seed=1, tour="random"),
    "C4": dict(n=33810, coords="lattice", seed=1, tour="random"),
    "C5": dict(n=85900, coords="lattice", seed=1, tour="random"),
}


def config_instance(name: str, tour_kind: str | None = None):
    """(coords int32[n,2], tour int32[n]) for a named config."""
    c = CONFIGS[name]
    coords = make_coords(c["coords"], c["n"], c["seed"])
    tour = make_tour(tour_kind or c["tour"], coords, c["seed"])
    return coords, tour
