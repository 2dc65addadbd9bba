"""Exhaustive pin: the oracle's nint over all 2^31-ish reachable s (tests/exhaustive_nint.c)."""
import os
import subprocess

import oracle

HERE = os.path.dirname(os.path.abspath(__file__))


def test_nint_exhaustive_all_reachable_s(tmp_path):
    lib = oracle.build()
    exe = tmp_path / "exh"
    subprocess.check_call(["gcc", "-O2", "-fopenmp", "-o", str(exe), os.path.join(HERE, "exhaustive_nint.c"),
                           lib, "-Wl,-rpath," + os.path.dirname(lib), "-lm"])
    out = subprocess.run([str(exe)], capture_output=True, text=True, timeout=600)
    checked, bad = map(int, out.stdout.split())
    assert bad == 0 and checked == 2 * 32767 * 32767 + 1
