"""Write golden local-search results for configs too slow for a live oracle run.

Calls ONLY oracle/ (and the seeded generators in inputs.py); never the CUDA path.

Usage:
  python tests/golden/make_golden.py C3 [--coords lattice] [--tour random|hilbert|mf] [--variant V]

Variants (the local search the golden records):
  2opt     best-improvement 2-opt, plain all-pairs oracle (oracle.local_search)
  radius   best-improvement 2-opt, exact radius-pruned oracle (oracle.radius_local_search;
           identical result by the lemma of SURVEY.md §8(c), pinned in tests/test_oracle_radius.py)
  first    first improvement (reading R20), exact radius-pruned oracle
  25opt    2.5-opt (reading R19), exact radius-pruned oracle
  knnK     the K-nearest-neighbour pruned neighbourhood (reading R18), oracle.pruned_local_search
  oropt    Or-opt (reading R21), plain oracle (oracle.local_search_or)

Output: tests/golden/ls_<variant>_<config>_<coords>_<tour>_s<seed>.npz (the 2opt variant
keeps its round-1 name ls_<config>_<coords>_<tour>_s<seed>.npz) with
  start (int32[n], the start tour; for --tour mf the oracle's Multiple Fragment tour),
  tour (int32[n]), length, iterations, status, trace (int64[it, 3 or 4] = i, j, delta[, type]),
  oracle_seconds, oracle_threads, variant.
"""
import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_ipps_rockis13_b200 import inputs  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))


def golden_path(config: str, coords: str, tour: str, seed: int, variant: str) -> str:
    if variant == "2opt":
        return os.path.join(HERE, f"ls_{config}_{coords}_{tour}_s{seed}.npz")
    return os.path.join(HERE, f"ls_{variant}_{config}_{coords}_{tour}_s{seed}.npz")


def start_tour(kind: str, coords: np.ndarray, seed: int) -> np.ndarray:
    if kind == "mf":
        return oracle.mf_tour(coords)
    return inputs.make_tour(kind, coords, seed)


def run(variant: str, coords: np.ndarray, tour: np.ndarray):
    cap = 40 * coords.shape[0] + 1000
    if variant == "2opt":
        return oracle.local_search(coords, tour, trace_cap=cap)
    if variant == "radius":
        return oracle.radius_local_search(coords, tour, trace_cap=cap)
    if variant == "first":
        return oracle.radius_local_search(coords, tour, trace_cap=cap, first=True)
    if variant == "25opt":
        return oracle.radius_local_search(coords, tour, trace_cap=cap, node_insertion=True)
    if variant.startswith("knn"):
        return oracle.pruned_local_search(coords, tour, int(variant[3:]), trace_cap=cap)
    if variant == "oropt":
        return oracle.local_search_or(coords, tour, trace_cap=cap)
    raise ValueError(variant)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--coords", default=None)
    ap.add_argument("--tour", default=None)
    ap.add_argument("--seed", type=int, default=None)
    ap.add_argument("--variant", default="2opt", help="comma-separated list")
    a = ap.parse_args()
    c = dict(inputs.CONFIGS[a.config])
    kind = a.coords or c["coords"]
    tk = a.tour or c["tour"]
    seed = a.seed if a.seed is not None else c["seed"]
    coords = inputs.make_coords(kind, c["n"], seed)
    t0 = time.time()
    tour = start_tour(tk, coords, seed)
    t_start = time.time() - t0
    print(f"{a.config} {tk} start: {t_start:.1f}s", flush=True)
    for variant in a.variant.split(","):
        t0 = time.time()
        res = run(variant, coords, tour)
        dt = time.time() - t0
        out = golden_path(a.config, kind, tk, seed, variant)
        np.savez_compressed(out, start=tour, tour=res["tour"], length=res["length"], iterations=res["iterations"],
                            status=res["status"], trace=res["trace"].astype(np.int64),
                            oracle_seconds=dt, start_seconds=t_start, oracle_threads=oracle.num_threads(),
                            variant=variant)
        print(out, res["length"], res["iterations"], f"{dt:.1f}s", oracle.num_threads(), "threads", flush=True)

if __name__ == "__main__":
    main()
