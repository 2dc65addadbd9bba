"""The bench's timed step alone, for one-configuration ncu launch lists:
    python tools/bench_step.py [CFG] [TILE_BOUNDS] [STEPS]
loads the seeded tour from device memory and runs one iteration (sweep + apply)
per step, exactly as bench.py's `value` loop (defaults: C5, bounds 0, 5 steps)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
bounds = int(sys.argv[2]) if len(sys.argv) > 2 else 0
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
coords, tour = inputs.config_instance(cfg, "random")
with tsp2opt.TSP2Opt(coords) as g:
    g.set_option(tsp2opt.OPT_TILE_BOUNDS, bounds)
    d_tour = torch.from_numpy(tour).cuda()
    for _ in range(steps):
        g.set_tour_device_async(d_tour.data_ptr())
        g.iterate_async(1)
    print(g.sync(), flush=True)
