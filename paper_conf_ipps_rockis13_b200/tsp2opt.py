"""Thin ctypes binding of libtsp2opt.so (include/tsp2opt.h).

Argument marshalling only: every step of the 2-opt path runs in the library's
CUDA kernels.  There is no CPU fallback: if the shared library is missing or
no CUDA device is present, calls raise.  Function names mirror the C ABI
without the `tsp2opt_` prefix; `TSP2Opt` is a convenience wrapper that owns a
handle.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from ._build import LIB as _DEFAULT_LIB

LIB = os.environ.get("TSP2OPT_LIB", _DEFAULT_LIB)  # override: an alternative in-tree build (experiments)

OK, MAXITER = 0, 1
EINVAL, ERANGE, ENOTPERM, ESTATE, ECUDA, ENCCL, ENOMEM = -1, -2, -3, -4, -5, -6, -7
NCCL_ID_BYTES = 128
MAX_ITERS_UNBOUNDED = (1 << 63) - 1

_lib = None


class TSP2OptError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        msg = _L().tsp2opt_strerror(code).decode()
        extra = _L().tsp2opt_last_error().decode()
        super().__init__(f"{where}: {msg} ({code})" + (f" [{extra}]" if extra else ""))


def _L():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            raise RuntimeError(
                f"{LIB} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                "(no CPU fallback exists)")
        lib = ctypes.CDLL(LIB)
        P, I32, I64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        pI32, pI64 = ctypes.POINTER(I32), ctypes.POINTER(I64)
        sig = {
            "tsp2opt_create": ([P, I32, ctypes.POINTER(P)], I32),
            "tsp2opt_create_sharded": ([P, I32, I32, I32, P, ctypes.POINTER(P)], I32),
            "tsp2opt_nccl_unique_id": ([P], I32),
            "tsp2opt_create_sharded_p2p": ([P, I32, I32, I32, ctypes.POINTER(P)], I32),
            "tsp2opt_p2p_export": ([P, P], I32),
            "tsp2opt_p2p_connect": ([P, P], I32),
            "tsp2opt_destroy": ([P], None),
            "tsp2opt_set_stream": ([P, P], I32),
            "tsp2opt_set_tour": ([P, P], I32),
            "tsp2opt_set_tour_device_async": ([P, P], I32),
            "tsp2opt_best_move": ([P, P, pI32, pI32, pI32], I32),
            "tsp2opt_apply": ([P, I32, I32], I32),
            "tsp2opt_iterate_async": ([P, I32], I32),
            "tsp2opt_sync": ([P, pI64, pI64, pI32, pI32, pI32, pI32], I32),
            "tsp2opt_local_search": ([P, P, I64, pI64, pI64], I32),
            "tsp2opt_get_tour": ([P, P, pI64], I32),
            "tsp2opt_debug_set_shard": ([P, I32, I32], I32),
            "tsp2opt_set_option": ([P, I32, I64], I32),
            "tsp2opt_get_trace": ([P, P, I64, pI64], I32),
            "tsp2opt_get_trace_typed": ([P, P, I64, pI64], I32),
            "tsp2opt_best_move_typed": ([P, P, pI32, pI32, pI32, pI32], I32),
            "tsp2opt_apply_typed": ([P, I32, I32, I32], I32),
            "tsp2opt_ils": ([P, P, I64, ctypes.c_uint64, pI64, P], I32),
            "tsp2opt_batch_local_search": ([P, I32, I32, P, I64, P, P], I32),
            "tsp2opt_mf_tour": ([P, P, pI64, P], I32),
            "tsp2opt_batch_local_search_async": ([P, I32, I32, P, I64, P, P, P], I32),
            "tsp2opt_batch_ils": ([P, I32, I32, P, I64, P, P, P], I32),
            "tsp2opt_batch_ils_async": ([P, I32, I32, P, I64, P, P, P, P], I32),
            "tsp2opt_oropt_local_search": ([P, I32, P, I64, pI64, pI64, P, I64], I32),
            "tsp2opt_oropt_best_move": ([P, I32, P, pI32, pI32, pI32, pI32], I32),
            "tsp2opt_oropt_config": ([I32, I32], I32),
            "tsp2opt_plan_shard": ([I32, I32, I32, pI32, pI32, pI32, P, I64, pI64, pI64], I32),
            "tsp2opt_get_geometry": ([P, pI32, pI32, pI32, pI64, pI64], I32),
            "tsp2opt_selftest": ([pI64, pI64, pI64, pI64], I32),
            "tsp2opt_profile": ([P, I32], I32),
            "tsp2opt_profile_read": ([P, ctypes.POINTER(ctypes.c_double), pI64], I32),
            "tsp2opt_launch_count": ([], I64),
            "tsp2opt_debug_stats": ([pI64, I32], I32),
            "tsp2opt_debug_phases": ([P, I32], I32),
            "tsp2opt_selftest_sqrt": ([ctypes.POINTER(ctypes.c_double), pI32], I32),
            "tsp2opt_strerror": ([I32], ctypes.c_char_p),
            "tsp2opt_last_error": ([], ctypes.c_char_p),
        }
        for name, (args, res) in sig.items():
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = res
        _lib = lib
    return _lib


def exported_symbols():
    """Names of the C-ABI entry points the binding expects (all declared in include/tsp2opt.h)."""
    _L()
    return [n for n in dir(_lib) if n.startswith("tsp2opt_")]


def _check(code: int, where: str) -> int:
    if code < 0:
        raise TSP2OptError(code, where)
    return code


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


# ----------------------------------------------------------------------------- C-ABI mirrors

def create(coords) -> ctypes.c_void_p:
    xy = _i32(coords).reshape(-1)
    h = ctypes.c_void_p()
    _check(_L().tsp2opt_create(_ptr(xy), xy.size // 2, ctypes.byref(h)), "tsp2opt_create")
    return h


def create_sharded(coords, rank: int, world: int, nccl_id: bytes | None) -> ctypes.c_void_p:
    xy = _i32(coords).reshape(-1)
    h = ctypes.c_void_p()
    idbuf = None if nccl_id is None else ctypes.create_string_buffer(bytes(nccl_id), NCCL_ID_BYTES)
    _check(_L().tsp2opt_create_sharded(_ptr(xy), xy.size // 2, rank, world, idbuf, ctypes.byref(h)),
           "tsp2opt_create_sharded")
    return h


P2P_HANDLE_BYTES = 64


def create_sharded_p2p(coords, rank: int, world: int) -> ctypes.c_void_p:
    """Sharded handle with the peer-memory exchange (tsp2opt_create_sharded_p2p)."""
    xy = _i32(coords).reshape(-1)
    h = ctypes.c_void_p()
    _check(_L().tsp2opt_create_sharded_p2p(_ptr(xy), xy.size // 2, rank, world, ctypes.byref(h)),
           "tsp2opt_create_sharded_p2p")
    return h


def p2p_export(h) -> bytes:
    buf = ctypes.create_string_buffer(P2P_HANDLE_BYTES)
    _check(_L().tsp2opt_p2p_export(h, buf), "tsp2opt_p2p_export")
    return buf.raw


def p2p_connect(h, handles) -> None:
    blob = b"".join(handles)
    buf = ctypes.create_string_buffer(blob, len(blob))
    _check(_L().tsp2opt_p2p_connect(h, buf), "tsp2opt_p2p_connect")


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(NCCL_ID_BYTES)
    _check(_L().tsp2opt_nccl_unique_id(buf), "tsp2opt_nccl_unique_id")
    return buf.raw


def destroy(h) -> None:
    _L().tsp2opt_destroy(h)


def set_stream(h, stream_handle: int | None) -> None:
    _check(_L().tsp2opt_set_stream(h, ctypes.c_void_p(stream_handle or 0)), "tsp2opt_set_stream")


def set_tour(h, tour) -> None:
    t = _i32(tour)
    _check(_L().tsp2opt_set_tour(h, _ptr(t)), "tsp2opt_set_tour")


def set_tour_device_async(h, device_ptr: int) -> None:
    _check(_L().tsp2opt_set_tour_device_async(h, ctypes.c_void_p(device_ptr)), "tsp2opt_set_tour_device_async")


def best_move(h, tour=None):
    i, j, d = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    if tour is None:
        tp = None
    else:
        t = _i32(tour)
        tp = _ptr(t)
    _check(_L().tsp2opt_best_move(h, tp, ctypes.byref(i), ctypes.byref(j), ctypes.byref(d)), "tsp2opt_best_move")
    return i.value, j.value, d.value


def apply(h, i: int, j: int) -> None:
    _check(_L().tsp2opt_apply(h, int(i), int(j)), "tsp2opt_apply")


def best_move_typed(h, tour=None):
    """(i, j, type, delta): the best move with its type (2.5-opt handles; type 0 otherwise)."""
    i, j, t, d = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    if tour is None:
        tp = None
    else:
        tt = _i32(tour)
        tp = _ptr(tt)
    _check(_L().tsp2opt_best_move_typed(h, tp, ctypes.byref(i), ctypes.byref(j), ctypes.byref(t), ctypes.byref(d)),
           "tsp2opt_best_move_typed")
    return i.value, j.value, t.value, d.value


def apply_typed(h, i: int, j: int, typ: int) -> None:
    _check(_L().tsp2opt_apply_typed(h, int(i), int(j), int(typ)), "tsp2opt_apply_typed")


def iterate_async(h, count: int) -> None:
    _check(_L().tsp2opt_iterate_async(h, int(count)), "tsp2opt_iterate_async")


def sync(h) -> dict:
    it, L = ctypes.c_int64(), ctypes.c_int64()
    cv, li, lj, ld = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    _check(_L().tsp2opt_sync(h, ctypes.byref(it), ctypes.byref(L), ctypes.byref(cv), ctypes.byref(li),
                             ctypes.byref(lj), ctypes.byref(ld)), "tsp2opt_sync")
    return dict(iterations=it.value, length=L.value, converged=cv.value, last_move=(li.value, lj.value, ld.value))


def local_search(h, tour, max_iters: int | None = None):
    """Returns dict(tour, length, iterations, status) with status OK (0) or MAXITER (1)."""
    t = np.array(tour, dtype=np.int32, copy=True)
    L, it = ctypes.c_int64(), ctypes.c_int64()
    mi = MAX_ITERS_UNBOUNDED if max_iters is None else int(max_iters)
    st = _check(_L().tsp2opt_local_search(h, _ptr(t), mi, ctypes.byref(L), ctypes.byref(it)), "tsp2opt_local_search")
    return dict(tour=t, length=L.value, iterations=it.value, status=st)


def mf_tour(h, n: int):
    """Multiple Fragment (greedy) start tour on the device; it becomes the current tour."""
    t = np.zeros(n, dtype=np.int32)
    L = ctypes.c_int64()
    r = ctypes.c_int32()
    _check(_L().tsp2opt_mf_tour(h, _ptr(t), ctypes.byref(L), ctypes.byref(r)), "tsp2opt_mf_tour")
    return dict(tour=t, length=L.value, rounds=r.value)


def local_search_current(h, max_iters: int | None = None):
    """Local search from the handle's current tour (tour == NULL); the result stays on the device."""
    L, it = ctypes.c_int64(), ctypes.c_int64()
    mi = MAX_ITERS_UNBOUNDED if max_iters is None else int(max_iters)
    st = _check(_L().tsp2opt_local_search(h, None, mi, ctypes.byref(L), ctypes.byref(it)), "tsp2opt_local_search")
    return dict(length=L.value, iterations=it.value, status=st)


def oropt_local_search(coords, tour, max_iters: int | None = None, trace_cap: int = 0):
    """Or-opt local search (reading R21), stateless: coords int32[n, 2], tour int32[n] ->
    dict(tour, length, iterations, status, trace int32[k, 4] rows (i, j, delta, type))."""
    xy = _i32(coords)
    n = xy.shape[0]
    t = np.array(tour, dtype=np.int32, copy=True).reshape(n)
    tr = np.zeros((max(trace_cap, 1), 4), dtype=np.int32)
    L, it = ctypes.c_int64(), ctypes.c_int64()
    mi = MAX_ITERS_UNBOUNDED if max_iters is None else int(max_iters)
    st = _check(_L().tsp2opt_oropt_local_search(_ptr(xy), n, _ptr(t), mi, ctypes.byref(L), ctypes.byref(it),
                                                _ptr(tr) if trace_cap > 0 else None, int(trace_cap)),
                "tsp2opt_oropt_local_search")
    return dict(tour=t, length=L.value, iterations=it.value, status=st, trace=tr[: min(it.value, trace_cap)].copy())


def oropt_config(filter: int = -1, naive: int = 0) -> None:
    """Or-opt kernel selection (no result depends on it): filter -1 by size, 0 off, 1 on;
    naive 1 selects the one-thread-per-cell kernel."""
    _check(_L().tsp2opt_oropt_config(int(filter), int(naive)), "tsp2opt_oropt_config")


def oropt_best_move(coords, tour):
    """(i, j, type, delta) of the best Or-opt move of `tour` (one device sweep)."""
    xy = _i32(coords)
    n = xy.shape[0]
    t = np.ascontiguousarray(tour, dtype=np.int32).reshape(n)
    i, j, ty, d = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    _check(_L().tsp2opt_oropt_best_move(_ptr(xy), n, _ptr(t), ctypes.byref(i), ctypes.byref(j), ctypes.byref(ty),
                                        ctypes.byref(d)), "tsp2opt_oropt_best_move")
    return i.value, j.value, ty.value, d.value


def batch_local_search(coords, tours, max_iters: int | None = None):
    """coords int32[B, n, 2], tours int32[B, n] -> dict(tours, lengths, iterations) (one CTA per instance)."""
    xy = _i32(coords)
    B, n = xy.shape[0], xy.shape[1]
    t = np.array(tours, dtype=np.int32, copy=True).reshape(B, n)
    L = np.zeros(B, dtype=np.int64)
    it = np.zeros(B, dtype=np.int64)
    mi = MAX_ITERS_UNBOUNDED if max_iters is None else int(max_iters)
    _check(_L().tsp2opt_batch_local_search(_ptr(xy), n, B, _ptr(t), mi, _ptr(L), _ptr(it)),
           "tsp2opt_batch_local_search")
    return dict(tours=t, lengths=L, iterations=it)


def batch_local_search_async(d_coords: int, n: int, batch: int, d_tours: int, d_lengths: int, d_iters: int,
                             max_iters: int | None = None, stream: int = 0):
    """Device-pointer form (raw addresses, e.g. torch tensor.data_ptr()); see include/tsp2opt.h."""
    mi = MAX_ITERS_UNBOUNDED if max_iters is None else int(max_iters)
    _check(_L().tsp2opt_batch_local_search_async(ctypes.c_void_p(d_coords), n, batch, ctypes.c_void_p(d_tours), mi,
                                                 ctypes.c_void_p(d_lengths), ctypes.c_void_p(d_iters),
                                                 ctypes.c_void_p(stream)), "tsp2opt_batch_local_search_async")


def batch_ils(coords, tours, iterations: int, seeds, history: bool = True):
    """Batched Iterated Local Search, one replica per CTA: coords int32[B, n, 2],
    tours int32[B, n], seeds uint64[B] -> dict(tours, lengths[, history int64[B, iterations+1]])."""
    xy = _i32(coords)
    B, n = xy.shape[0], xy.shape[1]
    t = np.array(tours, dtype=np.int32, copy=True).reshape(B, n)
    sd = np.ascontiguousarray(np.asarray(seeds, dtype=np.uint64).reshape(B))
    L = np.zeros(B, dtype=np.int64)
    hist = np.zeros((B, int(iterations) + 1), dtype=np.int64) if history else None
    _check(_L().tsp2opt_batch_ils(_ptr(xy), n, B, _ptr(t), int(iterations), _ptr(sd), _ptr(L),
                                  _ptr(hist) if history else None), "tsp2opt_batch_ils")
    out = dict(tours=t, lengths=L)
    if history:
        out["history"] = hist
    return out


def batch_ils_async(d_coords: int, n: int, batch: int, d_tours: int, iterations: int, d_seeds: int, d_lengths: int,
                    d_history: int = 0, stream: int = 0):
    """Device-pointer form (raw addresses); see include/tsp2opt.h."""
    _check(_L().tsp2opt_batch_ils_async(ctypes.c_void_p(d_coords), n, batch, ctypes.c_void_p(d_tours),
                                        int(iterations), ctypes.c_void_p(d_seeds), ctypes.c_void_p(d_lengths),
                                        ctypes.c_void_p(d_history or None), ctypes.c_void_p(stream)),
           "tsp2opt_batch_ils_async")


def ils(h, tour, iterations: int, seed: int):
    """Iterated Local Search (Algorithm 1): dict(tour, length, lengths)."""
    t = np.array(tour, dtype=np.int32, copy=True)
    L = ctypes.c_int64()
    lengths = np.zeros(int(iterations) + 1, dtype=np.int64)
    _check(_L().tsp2opt_ils(h, _ptr(t), int(iterations), ctypes.c_uint64(seed & 0xFFFFFFFFFFFFFFFF), ctypes.byref(L),
                            _ptr(lengths)), "tsp2opt_ils")
    return dict(tour=t, length=L.value, lengths=lengths)


def get_tour(h, n: int):
    """(tour int32[n], length) of handle h (n = the handle's city count)."""
    t = np.empty(n, dtype=np.int32)
    L = ctypes.c_int64()
    _check(_L().tsp2opt_get_tour(h, _ptr(t), ctypes.byref(L)), "tsp2opt_get_tour")
    return t, L.value


OPT_TILE_BOUNDS, OPT_SEED, OPT_PERSISTENT, OPT_TRACE, OPT_NEIGHBOURS, OPT_NODE_INSERTION = 1, 2, 3, 4, 5, 6
OPT_FIRST_IMPROVEMENT = 7
MAX_NEIGHBOURS = 16  # TSP2OPT_MAX_NEIGHBOURS


def set_option(h, option: int, value: int) -> None:
    _check(_L().tsp2opt_set_option(h, int(option), int(value)), "tsp2opt_set_option")


def get_trace(h, cap: int) -> np.ndarray:
    """int32[count, 3] (i, j, delta) of the recorded moves (set_option(OPT_TRACE, cap) first)."""
    out = np.zeros((max(cap, 1), 3), dtype=np.int32)
    cnt = ctypes.c_int64()
    _check(_L().tsp2opt_get_trace(h, _ptr(out), int(cap), ctypes.byref(cnt)), "tsp2opt_get_trace")
    return out[: min(cnt.value, cap)].copy()


def get_trace_typed(h, cap: int) -> np.ndarray:
    """int32[count, 4] (i, j, delta, type) of the recorded moves."""
    out = np.zeros((max(cap, 1), 4), dtype=np.int32)
    cnt = ctypes.c_int64()
    _check(_L().tsp2opt_get_trace_typed(h, _ptr(out), int(cap), ctypes.byref(cnt)), "tsp2opt_get_trace_typed")
    return out[: min(cnt.value, cap)].copy()


def debug_set_shard(h, rank: int, world: int) -> None:
    _check(_L().tsp2opt_debug_set_shard(h, rank, world), "tsp2opt_debug_set_shard")


def plan_shard(n: int, rank: int, world: int) -> dict:
    """Host-only: geometry and tile list (int32[ntiles, 2] of (I0, J0)) of one shard."""
    R, w, tj = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    nt, pairs = ctypes.c_int64(), ctypes.c_int64()
    _check(_L().tsp2opt_plan_shard(n, rank, world, ctypes.byref(R), ctypes.byref(w), ctypes.byref(tj), None, 0,
                                   ctypes.byref(nt), ctypes.byref(pairs)), "tsp2opt_plan_shard")
    tiles = np.zeros((nt.value, 2), dtype=np.int32)
    _check(_L().tsp2opt_plan_shard(n, rank, world, None, None, None, _ptr(tiles), nt.value, ctypes.byref(nt),
                                   ctypes.byref(pairs)), "tsp2opt_plan_shard")
    return dict(rows=R.value, warps=w.value, tj=tj.value, ti=32 * R.value * w.value, tiles=tiles,
                pairs=pairs.value)


def get_geometry(h) -> dict:
    R, w, tj = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    tiles, pairs = ctypes.c_int64(), ctypes.c_int64()
    _check(_L().tsp2opt_get_geometry(h, ctypes.byref(R), ctypes.byref(w), ctypes.byref(tj), ctypes.byref(tiles),
                                     ctypes.byref(pairs)), "tsp2opt_get_geometry")
    return dict(rows=R.value, warps=w.value, tj=tj.value, tiles=tiles.value, pairs=pairs.value)


def selftest() -> dict:
    a, b, c, d = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    _check(_L().tsp2opt_selftest(ctypes.byref(a), ctypes.byref(b), ctypes.byref(c), ctypes.byref(d)),
           "tsp2opt_selftest")
    return dict(dist_violations=a.value, filter_violations=b.value, first_bad_s=c.value, first_bad_dxdy=d.value)


def profile(h, enable: bool) -> None:
    _check(_L().tsp2opt_profile(h, 1 if enable else 0), "tsp2opt_profile")


def profile_read(h):
    """(summed device ms of the recorded sweep launches, number of launches)."""
    ms, n = ctypes.c_double(), ctypes.c_int64()
    _check(_L().tsp2opt_profile_read(h, ctypes.byref(ms), ctypes.byref(n)), "tsp2opt_profile_read")
    return ms.value, n.value


def selftest_sqrt() -> dict:
    """Max relative error of the sweep's MUFU.SQRT over every float in [1, 2^31]; sqrt(0) == 0."""
    e, z = ctypes.c_double(), ctypes.c_int32()
    _check(_L().tsp2opt_selftest_sqrt(ctypes.byref(e), ctypes.byref(z)), "tsp2opt_selftest_sqrt")
    return dict(max_rel_err=e.value, zero_ok=bool(z.value))


def launch_count() -> int:
    return int(_L().tsp2opt_launch_count())


# ----------------------------------------------------------------------------- convenience wrapper

class TSP2Opt:
    """One library handle (one GPU / one rank)."""

    def __init__(self, coords, rank: int = 0, world: int = 1, nccl_id: bytes | None = None, p2p_allgather=None):
        """p2p_allgather: a callable bytes -> list of every rank's bytes (rank order), e.g. over
        torch.distributed; selects the peer-memory exchange instead of NCCL."""
        xy = _i32(coords).reshape(-1, 2)
        self.n = xy.shape[0]
        if p2p_allgather is not None:
            self.h = create_sharded_p2p(xy, rank, world)
            try:
                p2p_connect(self.h, p2p_allgather(p2p_export(self.h)))
            except Exception:
                destroy(self.h)
                self.h = None
                raise
        else:
            # world 1 with an NCCL id: a one-rank communicator (the sharded path on one GPU)
            self.h = create(xy) if (world == 1 and nccl_id is None) else create_sharded(xy, rank, world, nccl_id)

    def close(self):
        if self.h:
            destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_stream(self, stream_handle: int | None):
        set_stream(self.h, stream_handle)

    def set_tour(self, tour):
        set_tour(self.h, tour)

    def set_tour_device_async(self, device_ptr: int):
        set_tour_device_async(self.h, device_ptr)

    def best_move(self, tour=None):
        return best_move(self.h, tour)

    def apply(self, i, j):
        apply(self.h, i, j)

    def best_move_typed(self, tour=None):
        return best_move_typed(self.h, tour)

    def apply_typed(self, i, j, typ):
        apply_typed(self.h, i, j, typ)

    def get_trace_typed(self, cap: int):
        return get_trace_typed(self.h, cap)

    def iterate_async(self, count: int):
        iterate_async(self.h, count)

    def sync(self):
        return sync(self.h)

    def local_search(self, tour, max_iters=None):
        return local_search(self.h, tour, max_iters)

    def get_tour(self):
        return get_tour(self.h, self.n)

    def mf_tour(self):
        return mf_tour(self.h, self.n)

    def local_search_current(self, max_iters=None):
        return local_search_current(self.h, max_iters)

    def ils(self, tour, iterations: int, seed: int):
        return ils(self.h, tour, iterations, seed)

    def set_option(self, option: int, value: int):
        set_option(self.h, option, value)

    def get_trace(self, cap: int):
        return get_trace(self.h, cap)

    def debug_set_shard(self, rank, world):
        debug_set_shard(self.h, rank, world)

    def geometry(self):
        return get_geometry(self.h)

    def profile(self, enable: bool):
        profile(self.h, enable)

    def profile_read(self):
        return profile_read(self.h)


def debug_phases(reset: bool = True) -> list:
    """Phase clocks of the persistent incremental search (instrumented builds; -1 otherwise)."""
    out = np.zeros(16, dtype=np.int64)
    _check(_L().tsp2opt_debug_phases(_ptr(out), 1 if reset else 0), "tsp2opt_debug_phases")
    return out.tolist()


def debug_stats(reset: bool = True) -> dict:
    """Sweep counters of an instrumented build (TSP2OPT_STATS); -1 in product builds."""
    out = (ctypes.c_int64 * 4)()
    _check(_L().tsp2opt_debug_stats(out, 1 if reset else 0), "tsp2opt_debug_stats")
    return dict(warp_steps=out[0], slow_steps=out[1], exact_pairs=out[2], tiles_walked=out[3])
