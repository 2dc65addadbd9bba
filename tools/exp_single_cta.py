"""One instance: the batched one-CTA kernel (B = 1) vs the handle's local search, device-resident timing."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

for n in (100, 150, 200, 300, 500, 1002):
    c = inputs.make_coords("uniform", n, 1)
    t = inputs.random_tour(n, 1)
    dc = torch.from_numpy(np.ascontiguousarray(c.reshape(-1))).cuda()
    dl = torch.zeros(1, dtype=torch.int64, device="cuda")
    di = torch.zeros(1, dtype=torch.int64, device="cuda")
    best = 1e9
    for rep in range(5):
        dt_ = torch.from_numpy(t.copy()).cuda()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        tsp2opt.batch_local_search_async(dc.data_ptr(), n, 1, dt_.data_ptr(), dl.data_ptr(), di.data_ptr())
        torch.cuda.synchronize()
        best = min(best, time.perf_counter() - t0)
    with tsp2opt.TSP2Opt(c) as g:
        g.local_search(t)
        hb = 1e9
        for rep in range(5):
            t0 = time.perf_counter()
            r = g.local_search(t)
            hb = min(hb, time.perf_counter() - t0)
    print(json.dumps({"n": n, "batch1_s": best, "batch_iters": int(di.item()), "handle_s": hb,
                      "handle_iters": r["iterations"]}), flush=True)
