"""B200 (sm_100a) exhaustive best-improvement 2-opt (Rocki & Suda, IPDPSW 2013).

The hot path lives in libtsp2opt.so (csrc/, C ABI in include/tsp2opt.h);
`tsp2opt` is its ctypes binding (the .so is loaded on first use) and `inputs`
holds the seeded synthetic instance / start-tour generators.  See DESIGN.md.
"""
from . import inputs, tsp2opt  # noqa: F401

__all__ = ["inputs", "tsp2opt"]
