"""Build libtsp2opt.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

`python -m paper_conf_ipps_rockis13_b200._build [--variant NAME -DFOO=1 ...]`
builds an experimental variant libtsp2opt_<NAME>.so with extra nvcc defines
(selected at run time with TSP2OPT_LIB=<path>); the default build is the product.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libtsp2opt.so")
SOURCES = [os.path.join(CSRC, f) for f in ("tsp2opt_kernels.cu", "tsp2opt_batch.cu", "tsp2opt_mf.cu", "tsp2opt_pruned.cu", "tsp2opt_sweep25.cu", "tsp2opt_oropt.cu", "tsp2opt_p2p.cu",
                                                    "tsp2opt_api.cu")]
HEADERS = [os.path.join(CSRC, f) for f in ("tsp2opt_device.cuh", "tsp2opt_internal.h", "tsp2opt_sweep.cuh")] + [
    os.path.join(ROOT, "include", "tsp2opt.h")
]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale(lib: str) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    return any(os.path.getmtime(f) > t for f in SOURCES + HEADERS)


def build(force: bool = False, verbose: bool = False, variant: str | None = None, defines=()) -> str:
    lib = LIB if variant is None else os.path.join(PKG, f"libtsp2opt_{variant}.so")
    if not force and not _stale(lib):
        return lib
    tmp = lib + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-shared",
           "-Xptxas", "-v", *defines, "-I", os.path.join(ROOT, "include"), "-o", tmp, *SOURCES, "-lnccl"]
    res = subprocess.run(cmd, capture_output=True, text=True)
    log = os.path.join(PKG, "build.log" if variant is None else f"build_{variant}.log")
    with open(log, "w") as f:
        f.write(" ".join(cmd) + "\n" + res.stdout + res.stderr)
    if res.returncode != 0:
        raise RuntimeError("nvcc failed:\n" + res.stderr[-4000:])
    if verbose:
        print(res.stderr)
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    args = sys.argv[1:]
    variant = None
    if args[:1] == ["--variant"]:
        variant, args = args[1], args[2:]
    print(build(force=True, variant=variant, defines=args))
