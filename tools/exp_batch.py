"""Time the batched small-instance local search (NEXT-3): device-resident
(async API, CUDA events), host API end to end, and one handle per instance
run sequentially.  Prints one JSON line per (n, B)."""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402


def batch(kind, n, B, seed0=1):
    cs = np.stack([inputs.make_coords(kind, n, seed0 + b) for b in range(B)]).astype(np.int32)
    ts = np.stack([inputs.random_tour(n, seed0 + b) for b in range(B)]).astype(np.int32)
    return cs, ts


def device_time(cs, ts, reps=3):
    B, n = ts.shape
    dc = torch.from_numpy(cs).cuda()
    t0 = torch.from_numpy(ts).cuda()
    dl = torch.zeros(B, dtype=torch.int64, device="cuda")
    di = torch.zeros(B, dtype=torch.int64, device="cuda")
    st = torch.cuda.current_stream()
    best = 1e9
    for _ in range(reps):
        dt = t0.clone()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        tsp2opt.batch_local_search_async(dc.data_ptr(), n, B, dt.data_ptr(), dl.data_ptr(), di.data_ptr(),
                                         stream=st.cuda_stream)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / 1e3)
    return best, di.cpu().numpy()


cases = [("uniform", 100, 148), ("uniform", 100, 1184), ("uniform", 100, 4736), ("uniform", 100, 18944),
         ("uniform", 200, 4736), ("uniform", 1002, 148), ("uniform", 1002, 592)]
for kind, n, B in cases:
    cs, ts = batch(kind, n, B)
    tsp2opt.batch_local_search(cs[:2], ts[:2])
    dev_s, its = device_time(cs, ts)
    t0 = time.perf_counter()
    out = tsp2opt.batch_local_search(cs, ts)
    host_s = time.perf_counter() - t0
    k = min(B, 8)
    t1 = time.perf_counter()
    for b in range(k):
        with tsp2opt.TSP2Opt(cs[b]) as g:
            g.local_search(ts[b])
    ds = (time.perf_counter() - t1) / k
    pairs = float(its.sum() + B) * n * (n - 1) / 2  # sweeps x pairs (last sweep finds no move)
    print(json.dumps(dict(kind=kind, n=n, B=B, threads=os.environ.get("TSP2OPT_BATCH_THREADS", "auto"),
                          packed=os.environ.get("TSP2OPT_BATCH_PACKED", "auto"),
                          device_s=round(dev_s, 6), inst_per_s=round(B / dev_s, 1),
                          pairs_per_s=f"{pairs / dev_s:.3e}", host_api_s=round(host_s, 5),
                          mean_moves=float(out["iterations"].mean()),
                          single_handle_inst_per_s=round(1 / ds, 1))), flush=True)
