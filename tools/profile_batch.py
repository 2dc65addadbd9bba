"""One batched-LS launch for ncu: python tools/profile_batch.py N B [reps]"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

n, B = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 1
cs = np.stack([inputs.make_coords("uniform", n, 1 + b) for b in range(B)]).astype(np.int32)
ts = np.stack([inputs.random_tour(n, 1 + b) for b in range(B)]).astype(np.int32)
dc, t0 = torch.from_numpy(cs).cuda(), torch.from_numpy(ts).cuda()
dl = torch.zeros(B, dtype=torch.int64, device="cuda")
di = torch.zeros(B, dtype=torch.int64, device="cuda")
for _ in range(reps):
    dt = t0.clone()
    tsp2opt.batch_local_search_async(dc.data_ptr(), n, B, dt.data_ptr(), dl.data_ptr(), di.data_ptr(),
                                     stream=torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
print("moves", int(di.sum()))
