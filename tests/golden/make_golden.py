"""Write golden local-search results for configs too slow for a live oracle run.

Calls ONLY oracle/ (and the seeded generators in inputs.py); never the CUDA path.
Usage: python tests/golden/make_golden.py C3 [--kind lattice] [--tour random]
Output: tests/golden/ls_<config>_<coords>_<tour>_s<seed>.npz with
        tour (int32[n]), length, iterations, status, trace (int64[it,3] = i, j, delta).
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--coords", default=None)
    ap.add_argument("--tour", default=None)
    ap.add_argument("--seed", type=int, default=None)
    a = ap.parse_args()
    c = dict(inputs.CONFIGS[a.config])
    kind = a.coords or c["coords"]
    tk = a.tour or c["tour"]
    seed = a.seed if a.seed is not None else c["seed"]
    coords = inputs.make_coords(kind, c["n"], seed)
    tour = inputs.make_tour(tk, coords, seed)
    t0 = time.time()
    res = oracle.local_search(coords, tour, trace_cap=10 * c["n"] + 1000)
    dt = time.time() - t0
    out = os.path.join(os.path.dirname(os.path.abspath(__file__)),
                       f"ls_{a.config}_{kind}_{tk}_s{seed}.npz")
    np.savez_compressed(out, tour=res["tour"], length=res["length"], iterations=res["iterations"],
                        status=res["status"], trace=res["trace"].astype(np.int64),
                        oracle_seconds=dt, oracle_threads=oracle.num_threads())
    print(out, res["length"], res["iterations"], f"{dt:.1f}s", oracle.num_threads(), "threads")


if __name__ == "__main__":
    main()
