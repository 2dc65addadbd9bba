"""The sharded path on two or more GPUs (§VI "dividing the 2-opt task
between multiple devices"; north_star (d)).

Runs tests/multirank_worker.py under torch.distributed.run with one rank per
visible GPU (at least 2; on a one-GPU box the test is skipped -- the same code
path runs there through a one-rank NCCL communicator, tests/test_gpu_nccl1.py,
and the shard split through simulated shards, test_gpu_parity.py).  Every rank's
final tour, length, iteration count and whole move trace must be identical, and
equal to the golden local search the oracle wrote (tests/golden/, make_golden.py).
"""
import hashlib
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.multigpu]

HERE = os.path.dirname(os.path.abspath(__file__))


def _gpus():
    import torch
    return torch.cuda.device_count()


@pytest.mark.parametrize("items", ["C3:hilbert,C3:mf", "C4:hilbert,C4:mf", "C5:hilbert"])
def test_sharded_local_search_equals_golden(gpu, items):
    n = _gpus()
    if n < 2:
        pytest.skip(f"needs >= 2 GPUs ({n} visible); covered on one GPU by test_gpu_nccl1.py and simulated shards")
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.join(HERE, "multirank_worker.py"), items]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=1800)
    assert out.returncode == 0, out.stderr[-3000:]
    line = next(x for x in out.stdout.splitlines() if x.startswith("MULTIRANK "))
    for res in json.loads(line[len("MULTIRANK "):]):
        cfg, _, tk = res["item"].partition(":")
        ranks = res["ranks"]
        assert all(r == ranks[0] for r in ranks), ranks  # identical state on every rank
        g = np.load(os.path.join(HERE, "golden", f"ls_radius_{cfg}_lattice_{tk}_s1.npz"))
        k = int(g["iterations"])
        want_trace = hashlib.sha1(g["trace"][:k].astype(np.int64).tobytes()).hexdigest()
        want_tour = hashlib.sha1(g["tour"].astype(np.int32).tobytes()).hexdigest()
        r0 = ranks[0]
        assert (r0["iterations"], r0["length"], r0["status"]) == (k, int(g["length"]), 0)
        assert r0["trace"] == want_trace and r0["tour"] == want_tour
