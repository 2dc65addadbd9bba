"""C-ABI boundary checks that need no GPU: the library loads, exports every
function include/tsp2opt.h declares, and rejects bad arguments before any
device work."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

from paper_conf_ipps_rockis13_b200 import tsp2opt
from paper_conf_ipps_rockis13_b200._build import LIB, build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "tsp2opt.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(tsp2opt_\w+)\s*\(", src)))


def test_library_builds_and_exports_every_declared_symbol():
    build()
    names = declared_functions()
    assert len(names) >= 18
    out = subprocess.run(["nm", "-D", "--defined-only", LIB], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r" T (tsp2opt_\w+)", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    lib = tsp2opt._L()
    for n in names:
        assert getattr(lib, n) is not None


def test_no_torch_types_in_signatures():
    src = open(os.path.join(ROOT, "include", "tsp2opt.h")).read()
    body = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    assert "at::" not in body and "Tensor" not in body and "c10" not in body


def test_argument_validation_without_gpu():
    lib = tsp2opt._L()
    h = ctypes.c_void_p()
    assert lib.tsp2opt_create(None, 10, ctypes.byref(h)) == tsp2opt.EINVAL
    xy = np.zeros(20, np.int32)
    for n in (0, 1, 2, (1 << 22) + 1):
        assert lib.tsp2opt_create(xy.ctypes.data, n, ctypes.byref(h)) == tsp2opt.EINVAL
    bad = np.zeros(20, np.int32)
    bad[7] = 1 << 15
    assert lib.tsp2opt_create(bad.ctypes.data, 10, ctypes.byref(h)) == tsp2opt.ERANGE
    bad[7] = -1
    assert lib.tsp2opt_create(bad.ctypes.data, 10, ctypes.byref(h)) == tsp2opt.ERANGE
    assert lib.tsp2opt_create_sharded(xy.ctypes.data, 10, 2, 2, None, ctypes.byref(h)) == tsp2opt.EINVAL
    assert lib.tsp2opt_create_sharded(xy.ctypes.data, 10, 0, 2, None, ctypes.byref(h)) == tsp2opt.EINVAL
    assert lib.tsp2opt_best_move(None, None, None, None, None) == tsp2opt.EINVAL
    assert lib.tsp2opt_apply(None, 0, 1) == tsp2opt.EINVAL
    assert lib.tsp2opt_local_search(None, None, 0, None, None) == tsp2opt.EINVAL
    # batched entry: sizes, ranges and permutations are checked before any device work
    L = np.zeros(2, np.int64)
    xy2 = np.zeros((2, 10, 2), np.int32)
    t2 = np.tile(np.arange(10, dtype=np.int32), (2, 1))
    bls = lib.tsp2opt_batch_local_search
    assert bls(None, 10, 2, t2.ctypes.data, 5, L.ctypes.data, L.ctypes.data) == tsp2opt.EINVAL
    for n, b in ((2, 2), (4097, 1), (10, 0)):
        assert bls(xy2.ctypes.data, n, b, t2.ctypes.data, 5, L.ctypes.data, L.ctypes.data) == tsp2opt.EINVAL
    assert bls(xy2.ctypes.data, 10, 2, t2.ctypes.data, -1, L.ctypes.data, L.ctypes.data) == tsp2opt.EINVAL
    badxy = xy2.copy()
    badxy[1, 3, 0] = 1 << 15
    assert bls(badxy.ctypes.data, 10, 2, t2.ctypes.data, 5, L.ctypes.data, L.ctypes.data) == tsp2opt.ERANGE
    badt = t2.copy()
    badt[1, 4] = 5
    assert bls(xy2.ctypes.data, 10, 2, badt.ctypes.data, 5, L.ctypes.data, L.ctypes.data) == tsp2opt.ENOTPERM
    assert lib.tsp2opt_strerror(tsp2opt.ENOTPERM) == b"tour is not a permutation of 0..n-1"
    # Or-opt entries (reading R21): validated on the host before any device work
    orl, orb = lib.tsp2opt_oropt_local_search, lib.tsp2opt_oropt_best_move
    t1 = np.arange(10, dtype=np.int32)
    i32 = ctypes.c_int32()
    assert orl(None, 10, t1.ctypes.data, 5, None, None, None, 0) == tsp2opt.EINVAL
    for n in (2, (1 << 20) + 1):
        assert orl(xy.ctypes.data, n, t1.ctypes.data, 5, None, None, None, 0) == tsp2opt.EINVAL
    assert orl(xy.ctypes.data, 10, t1.ctypes.data, -1, None, None, None, 0) == tsp2opt.EINVAL
    assert orl(xy.ctypes.data, 10, t1.ctypes.data, 5, None, None, None, 3) == tsp2opt.EINVAL
    bad = np.zeros(20, np.int32)
    bad[3] = 1 << 15
    assert orl(bad.ctypes.data, 10, t1.ctypes.data, 5, None, None, None, 0) == tsp2opt.ERANGE
    bt = t1.copy()
    bt[2] = 3
    assert orl(xy.ctypes.data, 10, bt.ctypes.data, 5, None, None, None, 0) == tsp2opt.ENOTPERM
    assert orb(xy.ctypes.data, 10, bt.ctypes.data, *([ctypes.byref(i32)] * 4)) == tsp2opt.ENOTPERM
    assert orb(xy.ctypes.data, 10, t1.ctypes.data, None, None, None, None) == tsp2opt.EINVAL


def test_key_layout_constants_match_header():
    src = open(os.path.join(ROOT, "include", "tsp2opt.h")).read()
    assert "#define TSP2OPT_MAX_N (1 << 22)" in src
    assert "#define TSP2OPT_COORD_LIMIT (1 << 15)" in src
