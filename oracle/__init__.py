"""CPU oracle for exhaustive best-improvement 2-opt (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  It wraps oracle/tsp2opt_oracle.c
(plain C, int64, OpenMP over the j loop) via ctypes and shares no code with
the CUDA path in paper_conf_ipps_rockis13_b200/.

Functions mirror the C file; each cites the passage it follows there.
Parity pins: tests/test_oracle*.py (pruned neighbourhood: tests/test_oracle_pruned.py).  `parity unpinned`: none.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tsp2opt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-o", tmp, _SRC, "-lm"]
        )
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            i64 = ctypes.c_int64
            p = ctypes.c_void_p
            lib.oracle_isqrt.argtypes = [i64]
            lib.oracle_isqrt.restype = i64
            lib.oracle_nint_sqrt.argtypes = [i64]
            lib.oracle_nint_sqrt.restype = i64
            lib.oracle_dist.argtypes = [i64, i64, i64, i64]
            lib.oracle_dist.restype = i64
            lib.oracle_tour_length.argtypes = [p, i64, p]
            lib.oracle_tour_length.restype = i64
            lib.oracle_delta.argtypes = [p, i64, p, i64, i64]
            lib.oracle_delta.restype = i64
            lib.oracle_cell.argtypes = [i64, i64]
            lib.oracle_cell.restype = i64
            lib.oracle_best_move.argtypes = [p, i64, p, p, p, p]
            lib.oracle_best_move.restype = None
            lib.oracle_best_move_tiles.argtypes = [p, i64, p, p, i64, i64, i64, p, p, p]
            lib.oracle_best_move_tiles.restype = None
            lib.oracle_apply.argtypes = [p, i64, i64]
            lib.oracle_apply.restype = None
            lib.oracle_local_search.argtypes = [p, i64, p, i64, p, p, p, i64]
            lib.oracle_local_search.restype = ctypes.c_int
            lib.oracle_double_bridge_cuts.argtypes = [i64, ctypes.c_uint64, i64, p, p, p]
            lib.oracle_double_bridge_cuts.restype = None
            lib.oracle_double_bridge.argtypes = [p, i64, i64, i64, i64, p]
            lib.oracle_double_bridge.restype = None
            lib.oracle_ils.argtypes = [p, i64, p, i64, ctypes.c_uint64, p, p]
            lib.oracle_ils.restype = None
            lib.oracle_mf_tour.argtypes = [p, i64, p]
            lib.oracle_mf_tour.restype = ctypes.c_int
            lib.oracle_knn.argtypes = [p, i64, i64, p]
            lib.oracle_knn.restype = None
            lib.oracle_pruned_best_move_plain.argtypes = [p, i64, p, p, i64, p, p, p]
            lib.oracle_pruned_best_move_plain.restype = None
            lib.oracle_pruned_best_move.argtypes = [p, i64, p, p, i64, p, p, p]
            lib.oracle_pruned_best_move.restype = None
            lib.oracle_pruned_first_move.argtypes = [p, i64, p, p, i64, p, p, p]
            lib.oracle_pruned_first_move.restype = None
            lib.oracle_pruned_local_search.argtypes = [p, i64, p, i64, i64, ctypes.c_int, p, p, p, i64]
            lib.oracle_pruned_local_search.restype = ctypes.c_int
            lib.oracle25_delta.argtypes = [p, i64, p, i64, i64, ctypes.c_int]
            lib.oracle25_delta.restype = i64
            lib.oracle25_best_move.argtypes = [p, i64, p, p, p, p, p]
            lib.oracle25_best_move.restype = None
            lib.oracle25_apply.argtypes = [p, i64, i64, ctypes.c_int]
            lib.oracle25_apply.restype = None
            lib.oracle25_local_search.argtypes = [p, i64, p, i64, p, p, p, i64]
            lib.oracle25_local_search.restype = ctypes.c_int
            lib.oracleor_delta.argtypes = [p, i64, p, i64, i64, ctypes.c_int]
            lib.oracleor_delta.restype = i64
            lib.oracleor_best_move.argtypes = [p, i64, p, p, p, p, p]
            lib.oracleor_best_move.restype = None
            lib.oracleor_apply.argtypes = [p, i64, i64, ctypes.c_int]
            lib.oracleor_apply.restype = None
            lib.oracleor_local_search.argtypes = [p, i64, p, i64, p, p, p, i64]
            lib.oracleor_local_search.restype = ctypes.c_int
            lib.oracle_first_move.argtypes = [p, i64, p, p, p, p]
            lib.oracle_first_move.restype = None
            lib.oracle_first_local_search.argtypes = [p, i64, p, i64, p, p, p, i64]
            lib.oracle_first_local_search.restype = ctypes.c_int
            lib.oracle_ils_mode.argtypes = [p, i64, p, i64, ctypes.c_uint64, ctypes.c_int, i64, p, p]
            lib.oracle_ils_mode.restype = None
            lib.oracle_radius_best_move.argtypes = [p, i64, p, ctypes.c_int, p, p, p, p]
            lib.oracle_radius_best_move.restype = None
            lib.oracle_radius_local_search.argtypes = [p, i64, p, i64, ctypes.c_int, p, p, p, i64]
            lib.oracle_radius_local_search.restype = ctypes.c_int
            lib.oracle_num_threads.argtypes = []
            lib.oracle_num_threads.restype = ctypes.c_int
            _lib = lib
    return _lib


def _xy(coords) -> np.ndarray:
    a = np.ascontiguousarray(np.asarray(coords, dtype=np.int32).reshape(-1, 2))
    return a


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def nint_sqrt(s: int) -> int:
    return int(_load().oracle_nint_sqrt(int(s)))


def isqrt(s: int) -> int:
    return int(_load().oracle_isqrt(int(s)))


def dist(a, b) -> int:
    return int(_load().oracle_dist(int(a[0]), int(a[1]), int(b[0]), int(b[1])))


def tour_length(coords, tour) -> int:
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    return int(_load().oracle_tour_length(_ptr(xy), xy.shape[0], _ptr(t)))


def delta(coords, tour, i: int, j: int) -> int:
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    return int(_load().oracle_delta(_ptr(xy), xy.shape[0], _ptr(t), i, j))


def cell(i: int, j: int) -> int:
    return int(_load().oracle_cell(i, j))


def best_move(coords, tour):
    """(i, j, delta) of the best 2-opt move of `tour` (Fig. 3 tie-break)."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    out = np.zeros(3, dtype=np.int64)
    _load().oracle_best_move(
        _ptr(xy), xy.shape[0], _ptr(t),
        _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]),
    )
    return int(out[0]), int(out[1]), int(out[2])


def best_move_tiles(coords, tour, tiles, ti: int, tj: int):
    """(i, j, delta): best move over the pairs of the given tiles only."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    tl = np.ascontiguousarray(np.asarray(tiles, dtype=np.int32).reshape(-1, 2))
    out = np.zeros(3, dtype=np.int64)
    _load().oracle_best_move_tiles(_ptr(xy), xy.shape[0], _ptr(t), _ptr(tl), tl.shape[0], ti, tj,
                                   _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]))
    return int(out[0]), int(out[1]), int(out[2])


def apply(tour, i: int, j: int) -> np.ndarray:
    """Return a copy of `tour` with positions i+1..j reversed."""
    t = np.array(tour, dtype=np.int32, copy=True)
    _load().oracle_apply(_ptr(t), i, j)
    return t


def local_search(coords, tour, max_iters: int = -1, trace_cap: int = 0):
    """Best-improvement 2-opt to a local minimum.

    Returns dict(tour, length, iterations, status, trace) where status is 0 at
    a local minimum and 1 when `max_iters` moves were applied and an improving
    move still remains; trace is int64[min(iterations, trace_cap), 3] (i, j, delta).
    """
    xy = _xy(coords)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(2, dtype=np.int64)
    tr = np.zeros((max(trace_cap, 1), 3), dtype=np.int64)
    st = _load().oracle_local_search(
        _ptr(xy), xy.shape[0], _ptr(t), int(max_iters),
        _ptr(out[0:1]), _ptr(out[1:2]), _ptr(tr) if trace_cap > 0 else None, int(trace_cap),
    )
    it = int(out[1])
    return dict(tour=t, length=int(out[0]), iterations=it, status=int(st),
                trace=tr[: min(it, trace_cap)].copy())


def double_bridge_cuts(n: int, seed: int, it: int):
    """(a, b, c) cut positions of ILS step `it` (reading R16)."""
    out = np.zeros(3, dtype=np.int64)
    _load().oracle_double_bridge_cuts(n, ctypes.c_uint64(seed & 0xFFFFFFFFFFFFFFFF), it,
                                      _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]))
    return int(out[0]), int(out[1]), int(out[2])


def double_bridge(tour, a: int, b: int, c: int) -> np.ndarray:
    t = np.ascontiguousarray(tour, dtype=np.int32)
    out = np.empty_like(t)
    _load().oracle_double_bridge(_ptr(t), t.size, a, b, c, _ptr(out))
    return out


def ils(coords, tour, iterations: int, seed: int, neighbours: int = 0, first: bool = False,
        node_insertion: bool = False):
    """Iterated Local Search (L10 Algorithm 1; readings R14-R16).
    Returns dict(tour, length, lengths) -- lengths[t] = best length after t steps.
    neighbours / first / node_insertion select the local search (R18 / R20 / R19)."""
    xy = _xy(coords)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(1, dtype=np.int64)
    lengths = np.zeros(iterations + 1, dtype=np.int64)
    if neighbours or first or node_insertion:
        if node_insertion and (neighbours or first):
            raise ValueError("2.5-opt combines with neither pruning nor first improvement")
        mode = 4 if node_insertion else (3 if neighbours and first else 1 if neighbours else 2)
        _load().oracle_ils_mode(_ptr(xy), xy.shape[0], _ptr(t), int(iterations),
                                ctypes.c_uint64(seed & 0xFFFFFFFFFFFFFFFF), mode, int(neighbours), _ptr(out),
                                _ptr(lengths))
        return dict(tour=t, length=int(out[0]), lengths=lengths)
    _load().oracle_ils(_ptr(xy), xy.shape[0], _ptr(t), int(iterations), ctypes.c_uint64(seed & 0xFFFFFFFFFFFFFFFF),
                       _ptr(out), _ptr(lengths))
    return dict(tour=t, length=int(out[0]), lengths=lengths)


def mf_tour(coords) -> np.ndarray:
    """Multiple Fragment (greedy) start tour (L22 §V; reading R17).  Plain: all
    C(n,2) edges sorted, 8 C(n,2) bytes of host memory (4.6 GB at C4, 29.5 GB at C5)."""
    xy = _xy(coords)
    t = np.zeros(xy.shape[0], dtype=np.int32)
    if _load().oracle_mf_tour(_ptr(xy), xy.shape[0], _ptr(t)) != 0:
        raise ValueError("oracle_mf_tour: n out of range [3, 2^22] or out of memory")
    return t


def _check_k(K: int) -> int:
    if int(K) < 1:
        raise ValueError("K must be >= 1")
    return int(K)


def knn(coords, K: int) -> np.ndarray:
    """N_K: int32[n, K] -- the K nearest cities of every city by (d, id), -1 pad
    (reading R18; L26 §VII "neighborhood pruning")."""
    xy = _xy(coords)
    K = _check_k(K)
    out = np.zeros((xy.shape[0], K), dtype=np.int32)
    _load().oracle_knn(_ptr(xy), xy.shape[0], K, _ptr(out))
    return out


def pruned_best_move(coords, tour, K: int, plain: bool = False, nbr=None):
    """(i, j, delta): best move of the K-nearest-neighbour pruned neighbourhood
    M_K (reading R18); plain=True scans all pairs with the membership test,
    else the O(nK) enumeration from the candidate lists."""
    xy = _xy(coords)
    K = _check_k(K)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    nb = knn(xy, K) if nbr is None else np.ascontiguousarray(nbr, dtype=np.int32)
    out = np.zeros(3, dtype=np.int64)
    fn = _load().oracle_pruned_best_move_plain if plain else _load().oracle_pruned_best_move
    fn(_ptr(xy), xy.shape[0], _ptr(t), _ptr(nb), K, _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]))
    return int(out[0]), int(out[1]), int(out[2])


def pruned_first_move(coords, tour, K: int, nbr=None):
    """(i, j, delta): the improving pair of M_K with the lowest Fig. 3 cell (readings R18 + R20)."""
    xy = _xy(coords)
    K = _check_k(K)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    nb = knn(xy, K) if nbr is None else np.ascontiguousarray(nbr, dtype=np.int32)
    out = np.zeros(3, dtype=np.int64)
    _load().oracle_pruned_first_move(_ptr(xy), xy.shape[0], _ptr(t), _ptr(nb), K, _ptr(out[0:1]), _ptr(out[1:2]),
                                     _ptr(out[2:3]))
    return int(out[0]), int(out[1]), int(out[2])


def pruned_local_search(coords, tour, K: int, max_iters: int = -1, trace_cap: int = 0, plain: bool = False,
                        first: bool = False):
    """Local search over M_K (best improvement, or first improvement with first=True);
    same return dict as local_search."""
    xy = _xy(coords)
    K = _check_k(K)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(2, dtype=np.int64)
    tr = np.zeros((max(trace_cap, 1), 3), dtype=np.int64)
    st = _load().oracle_pruned_local_search(
        _ptr(xy), xy.shape[0], _ptr(t), K, int(max_iters), (1 if plain else 0) | (2 if first else 0),
        _ptr(out[0:1]), _ptr(out[1:2]), _ptr(tr) if trace_cap > 0 else None, int(trace_cap),
    )
    it = int(out[1])
    return dict(tour=t, length=int(out[0]), iterations=it, status=int(st),
                trace=tr[: min(it, trace_cap)].copy())


def delta25(coords, tour, i: int, j: int, typ: int) -> int:
    """delta of 2.5-opt move (i, j, type) (reading R19); a huge value if not a move."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    return int(_load().oracle25_delta(_ptr(xy), xy.shape[0], _ptr(t), i, j, typ))


def best_move25(coords, tour):
    """(i, j, type, delta) of the best 2.5-opt move (reading R19: 2-opt plus node insertion)."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    out = np.zeros(4, dtype=np.int64)
    _load().oracle25_best_move(_ptr(xy), xy.shape[0], _ptr(t), _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]),
                               _ptr(out[3:4]))
    return int(out[0]), int(out[1]), int(out[2]), int(out[3])


def apply25(tour, i: int, j: int, typ: int) -> np.ndarray:
    t = np.array(tour, dtype=np.int32, copy=True)
    _load().oracle25_apply(_ptr(t), i, j, typ)
    return t


def local_search25(coords, tour, max_iters: int = -1, trace_cap: int = 0):
    """Best-improvement 2.5-opt local search; trace int64[k, 4] rows (i, j, delta, type)."""
    xy = _xy(coords)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(2, dtype=np.int64)
    tr = np.zeros((max(trace_cap, 1), 4), dtype=np.int64)
    st = _load().oracle25_local_search(_ptr(xy), xy.shape[0], _ptr(t), int(max_iters), _ptr(out[0:1]),
                                       _ptr(out[1:2]), _ptr(tr) if trace_cap > 0 else None, int(trace_cap))
    it = int(out[1])
    return dict(tour=t, length=int(out[0]), iterations=it, status=int(st), trace=tr[: min(it, trace_cap)].copy())


def delta_or(coords, tour, i: int, j: int, typ: int) -> int:
    """delta of Or-opt move (i, j, type) (reading R21); a huge value if not a move."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    return int(_load().oracleor_delta(_ptr(xy), xy.shape[0], _ptr(t), i, j, typ))


def best_move_or(coords, tour):
    """(i, j, type, delta) of the best Or-opt move (reading R21: 2-opt plus segment moves, L <= 3)."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    out = np.zeros(4, dtype=np.int64)
    _load().oracleor_best_move(_ptr(xy), xy.shape[0], _ptr(t), _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]),
                               _ptr(out[3:4]))
    return int(out[0]), int(out[1]), int(out[2]), int(out[3])


def apply_or(tour, i: int, j: int, typ: int) -> np.ndarray:
    t = np.array(tour, dtype=np.int32, copy=True)
    _load().oracleor_apply(_ptr(t), i, j, typ)
    return t


def local_search_or(coords, tour, max_iters: int = -1, trace_cap: int = 0):
    """Best-improvement Or-opt local search; trace int64[k, 4] rows (i, j, delta, type)."""
    xy = _xy(coords)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(2, dtype=np.int64)
    tr = np.zeros((max(trace_cap, 1), 4), dtype=np.int64)
    st = _load().oracleor_local_search(_ptr(xy), xy.shape[0], _ptr(t), int(max_iters), _ptr(out[0:1]),
                                       _ptr(out[1:2]), _ptr(tr) if trace_cap > 0 else None, int(trace_cap))
    it = int(out[1])
    return dict(tour=t, length=int(out[0]), iterations=it, status=int(st), trace=tr[: min(it, trace_cap)].copy())


def first_move(coords, tour):
    """(i, j, delta): the improving pair with the lowest Fig. 3 cell, else (0, 1, 0) (reading R20)."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    out = np.zeros(3, dtype=np.int64)
    _load().oracle_first_move(_ptr(xy), xy.shape[0], _ptr(t), _ptr(out[0:1]), _ptr(out[1:2]), _ptr(out[2:3]))
    return int(out[0]), int(out[1]), int(out[2])


def first_local_search(coords, tour, max_iters: int = -1, trace_cap: int = 0):
    """First-improvement 2-opt local search (reading R20); same return dict as local_search."""
    xy = _xy(coords)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(2, dtype=np.int64)
    tr = np.zeros((max(trace_cap, 1), 3), dtype=np.int64)
    st = _load().oracle_first_local_search(_ptr(xy), xy.shape[0], _ptr(t), int(max_iters), _ptr(out[0:1]),
                                           _ptr(out[1:2]), _ptr(tr) if trace_cap > 0 else None, int(trace_cap))
    it = int(out[1])
    return dict(tour=t, length=int(out[0]), iterations=it, status=int(st), trace=tr[: min(it, trace_cap)].copy())


def _radius_mode(first: bool, node_insertion: bool) -> int:
    if first and node_insertion:
        raise ValueError("the radius oracle has no first-improvement 2.5-opt")
    return 2 if node_insertion else (1 if first else 0)


def radius_best_move(coords, tour, first: bool = False, node_insertion: bool = False):
    """The exact radius-pruned sweep (SURVEY.md §8(c) lemma): equal to best_move (default),
    first_move (first=True) -> (i, j, delta), or best_move25 (node_insertion=True) ->
    (i, j, type, delta)."""
    xy = _xy(coords)
    t = np.ascontiguousarray(tour, dtype=np.int32)
    out = np.zeros(4, dtype=np.int64)
    mode = _radius_mode(first, node_insertion)
    _load().oracle_radius_best_move(_ptr(xy), xy.shape[0], _ptr(t), mode, _ptr(out[0:1]), _ptr(out[1:2]),
                                    _ptr(out[2:3]), _ptr(out[3:4]))
    if node_insertion:
        return int(out[0]), int(out[1]), int(out[2]), int(out[3])
    return int(out[0]), int(out[1]), int(out[3])


def radius_local_search(coords, tour, max_iters: int = -1, trace_cap: int = 0, first: bool = False,
                        node_insertion: bool = False):
    """Local search with the exact radius-pruned sweep; the same return dict (and trace
    rows) as local_search / first_local_search / local_search25."""
    xy = _xy(coords)
    t = np.array(tour, dtype=np.int32, copy=True)
    out = np.zeros(2, dtype=np.int64)
    w = 4 if node_insertion else 3
    tr = np.zeros((max(trace_cap, 1), w), dtype=np.int64)
    st = _load().oracle_radius_local_search(_ptr(xy), xy.shape[0], _ptr(t), int(max_iters),
                                            _radius_mode(first, node_insertion), _ptr(out[0:1]), _ptr(out[1:2]),
                                            _ptr(tr) if trace_cap > 0 else None, int(trace_cap))
    it = int(out[1])
    return dict(tour=t, length=int(out[0]), iterations=it, status=int(st), trace=tr[: min(it, trace_cap)].copy())


def num_threads() -> int:
    return int(_load().oracle_num_threads())
