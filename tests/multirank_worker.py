"""Worker of tests/test_gpu_multirank.py and tests/test_gpu_p2p.py, one process per
rank under torch.distributed.run.

Every rank builds a sharded handle (its equal-pair share of the tile list, one
allreduce-min of the packed key per sweep; §VI "dividing the 2-opt
task between multiple devices") and runs the full local search
with the move trace on.  --p2p: the exchange runs over peer-memory mailboxes
(tsp2opt_create_sharded_p2p; gloo only carries the 64-byte mailbox handles),
and ranks may share a GPU (rank r uses device r mod the visible count).  Rank 0 prints one JSON line with every rank's
(tour sha1, length, iterations, status, trace sha1) so the test can compare
them with each other and with the golden written by the oracle.
    torchrun --nproc-per-node N tests/multirank_worker.py CFG:START[,CFG:START...]
"""
import hashlib
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_ipps_rockis13_b200 import inputs, tsp2opt  # noqa: E402


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", rank))
    p2p, first = "--p2p" in sys.argv, "--first" in sys.argv
    torch.cuda.set_device(local % torch.cuda.device_count())
    if p2p:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    def allgather(b):
        out = [None] * world
        dist.all_gather_object(out, b)
        return out
    results = []
    for item in sys.argv[1].split(","):
        cfg, _, tk = item.partition(":")
        coords, tour = inputs.config_instance(cfg, "random" if tk == "mf" else tk)
        cap = 40 * len(coords)
        if p2p:
            handle = tsp2opt.TSP2Opt(coords, rank, world, p2p_allgather=allgather)
        else:
            obj = [tsp2opt.nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            handle = tsp2opt.TSP2Opt(coords, rank, world, obj[0])
        with handle as g:
            if tk == "mf":
                tour = g.mf_tour()["tour"]
            if first:
                g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
            g.set_option(tsp2opt.OPT_TRACE, cap)
            r = g.local_search(tour)
            tr = g.get_trace(cap)
        mine = {"tour": hashlib.sha1(r["tour"].astype(np.int32).tobytes()).hexdigest(),
                "trace": hashlib.sha1(tr.astype(np.int64).tobytes()).hexdigest(),
                "length": r["length"], "iterations": r["iterations"], "status": r["status"]}
        every = [None] * world
        dist.all_gather_object(every, mine)
        results.append({"item": item, "ranks": every})
    if rank == 0:
        print("MULTIRANK " + json.dumps(results), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
