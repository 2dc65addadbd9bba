#!/usr/bin/env python
"""Benchmark of the exhaustive best-improvement 2-opt hot path on B200.

Metric (BASELINE.json): 2-opt pair checks/sec (and time to local minimum) at
1/2/4/8 B200.  One timed STEP = one pass of every SURVEY.md §8(a) row over the
workload: load the tour from HBM (a2 reorder + a3 edges), the sweep over all
C(n,2) pairs (a4 + a5 reduce), the allreduce-min across ranks (a6, N > 1), the
segment-reversal apply (a7) and the loop-control state (a8).  Every step
reloads the same seeded random tour, so every step does identical work.

Workload (N=1 and N>1): config C5, n = 85900 pla-shaped lattice, random tour
(BASELINE.json configs[4]; the metric names 1/2/4/8 GPUs, which only the
sharded configs have).  `value` = C(n,2) * K / (max over ranks of the device
time of the K steps); `e2e` = the same through the C ABI with host buffers.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_rockis13_b200 import inputs  # noqa: E402

METRIC = "2-opt pair checks/sec and time-to-local-minimum at 1/2/4/8 B200 vs roofline"
UNIT = "pair checks/s"
PAIRS_PER_CLK_SM = 8  # north_star's per-pair model: ~2 distance evaluations (16 issue slots, 2 XU ops) per pair
ISSUE_PER_CLK_SM = 4  # warp-instruction issue slots per clock per SM (4 SMSPs) -- the sweep's real ceiling
N_SM = 148


def peaks():
    p = {}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
    except OSError:
        pass
    return p


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """SM clock and throttle reasons sampled (NVML, every ~2 ms) during the timed region."""

    REASONS = {  # nvmlClocksEventReason bits
        0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown", 0x4: "sw_power_cap",
        0x80: "hw_power_brake_slowdown",
    }

    def __init__(self, device: int):
        self.device = device
        self.samples = []
        self.reasons = set()
        self.run = False
        self.ok = False

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.device)
            self.max = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)
            return
        self.run = True
        self.t = threading.Thread(target=self._loop, daemon=True)
        self.t.start()

    def _loop(self):
        nv = self.nv
        while self.run:
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def stop(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "nvml")}
        self.run = False
        self.t.join(timeout=2)
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ----------------------------------------------------------------------------- distributed
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def l2_flush(buf):
    buf.add_(1)  # writes 256 MiB > 126 MB L2


# ----------------------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_rockis13_b200 import tsp2opt

    rank, world, local = dist_env()
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    p2p = args.exchange == "p2p"
    # --exchange p2p: the per-sweep MIN over peer-memory mailboxes; ranks may then share a
    # GPU (rank r on device r mod the visible count: a code-path check on a one-GPU box,
    # the ranks time-slice), and gloo carries only the host-side collectives
    torch.cuda.set_device(local % torch.cuda.device_count() if p2p else local)
    if world > 1:
        if p2p:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    hdev = "cpu" if p2p else "cuda"  # device of the tensors the host-side collectives reduce
    cfg = inputs.CONFIGS[args.config]
    n = cfg["n"]
    coords, tour = inputs.config_instance(args.config, args.tour)
    total_pairs = n * (n - 1) // 2

    g = sharded_handle(tsp2opt, coords, rank, world, p2p) if world > 1 else tsp2opt.TSP2Opt(coords)
    stream = torch.cuda.Stream()  # a real stream: events and the library's launches share it
    torch.cuda.set_stream(stream)
    g.set_stream(stream.cuda_stream)
    d_tour = torch.from_numpy(tour).cuda()
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
    torch.cuda.synchronize()

    def step():
        g.set_tour_device_async(d_tour.data_ptr())
        g.iterate_async(1)

    def timed_steps(nsteps, sample_clocks):
        """K device-timed steps (CUDA events on the library's stream, L2 flushed
        between steps outside the events); the sweep kernel timed separately."""
        for _ in range(args.warmup):
            step()
        s = g.sync()
        first = s["last_move"]
        sampler = ClockSampler(torch.cuda.current_device()) if sample_clocks else None
        if sampler:
            sampler.start()
        starts = [torch.cuda.Event(enable_timing=True) for _ in range(nsteps)]
        ends = [torch.cuda.Event(enable_timing=True) for _ in range(nsteps)]
        g.profile(True)
        launches0 = tsp2opt.launch_count()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        for k in range(nsteps):
            l2_flush(flush)  # between timed steps, outside the events
            starts[k].record(stream)
            step()
            ends[k].record(stream)
        torch.cuda.synchronize()
        nlaunch = tsp2opt.launch_count() - launches0
        if world > 1:
            dist.barrier()
        clk = sampler.stop() if sampler else None
        sms, sn = g.profile_read()
        g.profile(False)
        tot = sum(a.elapsed_time(b) for a, b in zip(starts, ends))
        s = g.sync()
        assert s["iterations"] == 1 and s["last_move"] == first, "steps must be identical"
        return tot, sms / max(sn, 1), nlaunch, clk, first

    # Headline: every pair tested individually (tile bounds off), DESIGN.md §7.
    g.set_option(tsp2opt.OPT_TILE_BOUNDS, 0)
    total_ms, sweep_avg_ms, launches, clocks, first_move = timed_steps(args.steps, True)
    # Same workload with the exact tile-level bounds on (the library default).
    g.set_option(tsp2opt.OPT_TILE_BOUNDS, 1)
    tb_total_ms, tb_sweep_ms, _, _, tb_move = timed_steps(max(3, args.steps // 2), False)
    assert tb_move == first_move
    g.set_option(tsp2opt.OPT_TILE_BOUNDS, 0)

    # e2e: same metric through the public C ABI with HOST buffers each step
    # (H2D of the tour, device sweep + apply, D2H of the move and the state).
    geo = g.geometry()
    g.set_stream(None)
    e2e_ms = []
    host_tour = torch.from_numpy(tour).pin_memory().numpy()  # the step's input in pinned host memory
    for k in range(max(2, args.steps // 2) + 1):
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        i, j, d = g.best_move(host_tour)
        if d < 0:
            g.apply(i, j)
        e2e_ms.append((time.perf_counter() - t0) * 1e3)
    e2e_ms = e2e_ms[1:]
    tb_steps = max(3, args.steps // 2)

    t = torch.tensor([total_ms, sweep_avg_ms, sum(e2e_ms), tb_total_ms, tb_sweep_ms], dtype=torch.float64,
                     device=hdev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms, sweep_avg_ms, e2e_total, tb_total_ms, tb_sweep_ms = t.tolist()

    ls = ils = batch = batch_ils = pruned = or25 = first = oropt = sharded = balance = None
    if world > 1 and not args.no_ls:  # collective: every rank runs it
        sharded = time_sharded_ls(tsp2opt, rank, world, args.sharded_config, p2p)
    if rank == 0 and world == 1 and not args.no_ls and args.balance_config:
        balance = shard_balance(tsp2opt, args.balance_config)
    if rank == 0 and world == 1 and not args.no_ls:
        ls = time_to_local_min(tsp2opt, args.ls_config, not args.no_cpu)
        pruned = time_pruned(tsp2opt, args.pruned_config, not args.no_cpu) if args.pruned_config else None
        or25 = time_25opt(tsp2opt, args.or25_config, not args.no_cpu) if args.or25_config else None
        first = time_first(tsp2opt, args.first_config) if args.first_config else None
        oropt = time_oropt(tsp2opt, args.oropt_config, not args.no_cpu) if args.oropt_config else None
        ils = time_ils(tsp2opt, args.ils_config) if args.ils_config else None
        batch = time_batch(tsp2opt, args.batch_config, not args.no_cpu) if args.batch_config else None
        batch_ils = time_batch_ils(tsp2opt, args.batch_ils_config, not args.no_cpu) if args.batch_ils_config else None

    if rank == 0:
        prof = ncu_profile_summary(args.config, args.tour)
        pk = peaks()
        sm_max = clocks.get("sm_max_mhz") or pk.get("sm_max_mhz") or 1965.0
        pair_peak = PAIRS_PER_CLK_SM * N_SM * sm_max * 1e6 * world  # north_star's per-pair model, all ranks
        pair_rate = geo["pairs"] * world / (sweep_avg_ms * 1e-3)  # pairs per second of sweep launch, all ranks
        value = total_pairs * args.steps / (total_ms * 1e-3)
        # Roofline: the sweep is issue-bound, so `frac` is the issue-slot
        # fraction -- the warp instructions ONE sweep launch executes (ncu, committed
        # profile of this workload) over the live launch time, against 4 warp-inst/clk/SM.
        issue_peak = ISSUE_PER_CLK_SM * N_SM * sm_max * 1e6  # warp-instructions/s per GPU
        winst = prof.get("warp_inst")  # one full single-GPU sweep; a rank's shard does its share of it
        if winst:
            winst *= geo["pairs"] / total_pairs
        issue_rate = winst / (sweep_avg_ms * 1e-3) if winst else None
        line = {
            "metric": METRIC,
            "value": value,
            "unit": UNIT,
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": total_ms / args.steps,
            "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak",
            "exchange": ("peer memory" if p2p else "NCCL") if world > 1 else None,
            "vs_baseline": None,
            "dtype": "int32+f32",
            "data": "synthetic",
            "config": {"workload": f"{args.config} n={n} {cfg['coords']} coords seed={cfg['seed']}, "
                                   f"{args.tour} tour; one step = load tour + sweep C(n,2) pairs + "
                                   f"{'allreduce-min + ' if world > 1 else ''}apply",
                       "n": n, "pairs_per_step": total_pairs, "l2": "flushed (256 MiB write) between timed steps",
                       "geometry": geo, "parallelism": f"tile-shard x{world}"},
            "roofline": {"bound": "alu", "achieved": issue_rate / 1e12 if issue_rate else None,
                         "peak": issue_peak / 1e12, "unit": "Twarp-inst/s",
                         "frac": issue_rate / issue_peak if issue_rate else None, "traffic": prof.get("traffic"),
                         "kernel": "sweep_kernel",
                         "peak_def": f"{ISSUE_PER_CLK_SM} warp-instructions/clk/SM (4 SMSPs x 1 issue) x {N_SM} SMs x "
                                     f"{sm_max:.0f} MHz: the sweep is issue-bound (DESIGN.md §5.4, §7)",
                         "achieved_def": "warp instructions per C5 sweep launch (ncu smsp__inst_executed.sum of the "
                                         "committed profile) / live sweep-launch time (CUDA events, this run)",
                         "warp_inst_per_launch": winst, "inst_per_pair": (32 * winst / geo["pairs"]) if winst else None,
                         "ncu_profile": prof.get("path"), "ncu_issue_active": prof.get("issue_util"),
                         "sweep_ms_avg": sweep_avg_ms, "sweep_share_of_step": sweep_avg_ms / (total_ms / args.steps),
                         "pair_rate": pair_rate / 1e9, "pair_rate_unit": "Gpair/s (all ranks)",
                         "model_ratio": pair_rate / pair_peak,
                         "model_def": f"pair rate / ({PAIRS_PER_CLK_SM} pairs/clk/SM x {N_SM} x {sm_max:.0f} MHz x "
                                      f"{world}), north_star's ~2 distance evaluations per pair; > 1 means fewer "
                                      "instructions per pair than that model, not above the hardware limit"},
            "e2e": {"value": total_pairs * len(e2e_ms) / (e2e_total * 1e-3), "unit": UNIT,
                    "h2d_bytes_per_step": 4 * n, "d2h_bytes_per_step": 2 * 64,
                    "api": "tsp2opt_best_move(pinned host tour) + tsp2opt_apply; wall clock per step, first step dropped"},
            "tile_bounds": {"value": total_pairs * tb_steps / (tb_total_ms * 1e-3), "unit": UNIT,
                            "ms_per_step": tb_total_ms / tb_steps, "sweep_ms_avg": tb_sweep_ms,
                            "note": "same steps with the exact tile-level bounding-box bound on (library default); "
                                    "pairs of a skipped tile are covered by one proof, not tested one by one"},
            "gpu_launches": launches,
            "clocks": clocks,
            "first_move": list(first_move),
        }
        if ls:
            line["time_to_local_minimum"] = ls
        if sharded:
            line["time_to_local_minimum_sharded"] = sharded
        if balance:
            line["shard_load_balance"] = balance
        if ils:
            line["ils"] = ils
        if pruned:
            line["pruned_local_search"] = pruned
        if or25:
            line["local_search_25opt"] = or25
        if first:
            line["local_search_first_improvement"] = first
        if oropt:
            line["local_search_oropt"] = oropt
        if batch:
            line["batch_local_search"] = batch
        if batch_ils:
            line["batch_ils"] = batch_ils
        if world == 1 and not args.no_cpu:
            line["cpu_baseline"] = cpu_baseline(args, coords, tour, total_pairs)
        print(json.dumps(line), flush=True)
    g.close()
    if world > 1:
        dist.destroy_process_group()


def ncu_profile_summary(cfg, tour):
    """DRAM traffic per launch and issue utilisation of the sweep kernel from the
    committed `ncu --set full` summary of this workload (profiles/, newest round)."""
    import glob
    paths = sorted(glob.glob(os.path.join(ROOT, "profiles", f"r*_sweep_{cfg}_{tour}_ncu.txt")))
    if not paths:
        return {}
    vals = {}
    for line in open(paths[-1]):
        if line.startswith("ipc_per_sm"):
            vals["ipc_per_sm"] = float(line.split()[3])
        elif line.startswith("warp_inst_total"):
            vals["warp_inst"] = float(line.split()[1])
        elif line.startswith(("dram_read", "dram_write")):
            name, num, unit = (line.split() + ["byte"])[:3]
            vals[name] = float(num) * {"Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "Gbyte": 1e9}.get(unit, 1.0)
    out = {"path": os.path.relpath(paths[-1], ROOT)}
    if "dram_read" in vals:
        out["traffic"] = vals["dram_read"] + vals.get("dram_write", 0.0)
    if "ipc_per_sm" in vals:
        out["issue_util"] = vals["ipc_per_sm"] / 4.0
    if "warp_inst" in vals:
        out["warp_inst"] = vals["warp_inst"]
    return out


def oracle_ttlm(name, tk, coords, tour):
    """The oracle's time to the same local minimum (Table II "Time to first
    minimum"; SURVEY §8(d) "full local search for C1-C3"): C1 and C2 run live on this
    box's host cores; C3-C5 are too slow for a bench run, so their figure is the
    oracle_seconds recorded by tests/golden/make_golden.py (labelled with its
    threads and, for C4 / C5, the exact radius-pruned oracle it used)."""
    import oracle

    n = len(coords)
    if n <= 2000:
        if tour is None:  # the Multiple Fragment start: the oracle's own (never the device's)
            tour = oracle.mf_tour(coords)
        t0 = time.perf_counter()
        r = oracle.local_search(coords, tour)
        return {"seconds": time.perf_counter() - t0, "iterations": r["iterations"], "length": r["length"],
                "cores": oracle.num_threads(), "kind": "oracle", "sample": "the whole local search, live"}
    gdir = os.path.join(ROOT, "tests", "golden")
    cands = [(f"ls_{name}_lattice_{tk}_s1.npz", "plain all-pairs oracle"),
             (f"ls_radius_{name}_lattice_{tk}_s1.npz", "exact radius-pruned oracle (SURVEY §8(c) lemma; same moves)")]
    for fname, what in cands:
        path = os.path.join(gdir, fname)
        if os.path.exists(path):
            g = np.load(path)
            return {"seconds": float(g["oracle_seconds"]), "iterations": int(g["iterations"]),
                    "length": int(g["length"]), "cores": int(g["oracle_threads"]), "kind": "oracle",
                    "sample": f"recorded by tests/golden/make_golden.py on the 8-core dev host, {what}"}
    return None


def time_to_local_min(tsp2opt, cfg_name, with_oracle=True):
    """Wall time of tsp2opt_local_search (host tour in, host tour out) per config.
    Start `mf`: the paper's Table II protocol (L22 "time needed from an initial
    solution based on the Multiple Fragment(Greedy) heuristic ... to the local
    minimum"): tsp2opt_mf_tour on the device, then the local search from it;
    both inside the timed region (coordinates already on the device).
    `pairs_covered_per_s` = C(n,2) x sweeps / time: with the tile bounds and the
    culled / incremental sweeps most pairs are covered by a tile-level proof, not
    tested one by one, so it is NOT a pair-check rate (that is the dense `value`)."""
    out = []
    for name in cfg_name.split(","):
        name, _, tk = name.partition(":")
        if tk == "mf":
            coords, _ = inputs.config_instance(name)
            with tsp2opt.TSP2Opt(coords) as g:
                g.mf_tour()  # warm-up (allocates the workspace)
                g.local_search_current(max_iters=2)
                t0 = time.perf_counter()
                m = g.mf_tour()
                t1 = time.perf_counter()
                r = g.local_search_current()
                t2 = time.perf_counter()
            n = len(coords)
            entry = {"config": name, "n": n, "start": "mf", "seconds": t2 - t0, "mf_seconds": t1 - t0,
                     "ls_seconds": t2 - t1, "mf_length": m["length"], "mf_rounds": m["rounds"],
                     "iterations": r["iterations"], "length": r["length"],
                     "us_per_move": 1e6 * (t2 - t1) / max(1, r["iterations"]),
                     "pairs_covered_per_s": (r["iterations"] + 1) * n * (n - 1) / 2 / (t2 - t1)}
            if with_oracle:
                o = oracle_ttlm(name, "mf", coords, None)
                if o:
                    entry["cpu_oracle"] = o
            out.append(entry)
            continue
        coords, tour = inputs.config_instance(name, tk or None)
        with tsp2opt.TSP2Opt(coords) as g:
            g.local_search(tour, max_iters=2)  # warm-up
            t0 = time.perf_counter()
            r = g.local_search(tour)
            dt = time.perf_counter() - t0
        n = len(tour)
        tk = tk or inputs.CONFIGS[name]["tour"]
        entry = {"config": name, "n": n, "start": tk, "seconds": dt,
                 "iterations": r["iterations"], "length": r["length"],
                 "us_per_move": 1e6 * dt / max(1, r["iterations"]),
                 "pairs_covered_per_s": (r["iterations"] + 1) * n * (n - 1) / 2 / dt}
        if with_oracle:
            o = oracle_ttlm(name, tk, coords, tour)
            if o:
                entry["cpu_oracle"] = o
        out.append(entry)
    return out


def sharded_handle(tsp2opt, coords, rank, world, p2p):
    """A sharded handle on every rank: NCCL (unique id broadcast by torch.distributed) or
    the peer-memory exchange (mailbox handles all-gathered)."""
    import torch.distributed as dist

    if p2p:
        def allgather(b):
            out = [None] * world
            dist.all_gather_object(out, b)
            return out
        return tsp2opt.TSP2Opt(coords, rank, world, p2p_allgather=allgather)
    obj = [tsp2opt.nccl_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    return tsp2opt.TSP2Opt(coords, rank, world, obj[0])


def time_sharded_ls(tsp2opt, rank, world, spec, p2p=False):
    """Time to local minimum on sharded handles (§VI "dividing the 2-opt task
    between multiple devices"): every rank runs tsp2opt_local_search on its
    tile shard with one allreduce-min per sweep.  seconds = max over ranks of each rank's
    wall time of the call, the ranks started together by a barrier.  Every rank's final
    tour must be identical (tour hash all-gathered) and equal to the length / move count
    a world-1 run reports (checked by tests/test_gpu_multirank.py)."""
    import hashlib

    import torch
    import torch.distributed as dist

    out = []
    for item in spec.split(","):
        if not item:
            continue
        name, _, tk = item.partition(":")
        coords, tour = inputs.config_instance(name, "random" if tk == "mf" else (tk or None))
        with sharded_handle(tsp2opt, coords, rank, world, p2p) as g:
            if tk == "mf":
                tour = g.mf_tour()["tour"]
            g.local_search(tour, max_iters=2)  # warm-up (graphs, NCCL channels)
            dist.barrier()
            t0 = time.perf_counter()
            r = g.local_search(tour)
            dt = time.perf_counter() - t0
        t = torch.tensor([dt], dtype=torch.float64, device="cpu" if p2p else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        h = hashlib.sha1(r["tour"].tobytes()).hexdigest()[:16]
        hs = [None] * world
        dist.all_gather_object(hs, (h, r["iterations"], r["length"]))
        n = len(coords)
        out.append({"config": name, "n": n, "start": tk or "random", "ranks": world, "seconds": t.item(),
                    "iterations": r["iterations"], "length": r["length"],
                    "us_per_move": 1e6 * t.item() / max(1, r["iterations"]),
                    "tours_agree": all(x == hs[0] for x in hs), "tour_sha1_16": h,
                    "exchange": "peer memory" if p2p else "NCCL",
                    "timing": "max over ranks of the per-rank wall time of tsp2opt_local_search"})
    return out


def shard_balance(tsp2opt, spec):
    """Load balance of the equal-pair LPT tile split, measured on ONE GPU:
    for world = 2, 4, 8 every shard r of the dense C4 / C5 sweep (random tour, tile bounds
    off, the bench's `value` workload) is timed alone with tsp2opt_debug_set_shard(r, world)
    and the library's CUDA events; reported as max / mean shard time.  The min over the
    shards' moves must equal the full sweep's move.  A load-balance check of the split,
    not a multi-GPU measurement."""
    out = []
    for name in spec.split(","):
        if not name:
            continue
        coords, tour = inputs.config_instance(name, "random")
        with tsp2opt.TSP2Opt(coords) as g:
            g.set_option(tsp2opt.OPT_TILE_BOUNDS, 0)
            full = g.best_move(tour)
            for world in (2, 4, 8):
                times, moves = [], []
                for r in range(world):
                    g.debug_set_shard(r, world)
                    g.best_move(tour)
                    g.profile(True)
                    for _ in range(3):
                        mv = g.best_move()
                    ms, k = g.profile_read()
                    g.profile(False)
                    times.append(ms / k)
                    moves.append(mv)
                g.debug_set_shard(0, 1)
                best = min(moves, key=lambda m: (m[2], m[1] * (m[1] - 1) // 2 + m[0]))
                out.append({"config": name, "world": world, "shard_ms": times,
                            "max_over_mean": max(times) / (sum(times) / world),
                            "min_of_shards_equals_full": best == full})
    return out


def time_pruned(tsp2opt, spec, with_oracle=True):
    """Neighbourhood-pruned 2-opt (TSP2OPT_OPT_NEIGHBOURS = K; SURVEY §8(f)
    NEXT-4, L26 §VII "neighborhood pruning ... at the cost of the quality";
    reading R18) from the Multiple Fragment start, `cfg:K` entries: MF tour,
    the local search over M_K, then the full neighbourhood continued from the
    pruned minimum to a full 2-opt local minimum (polish); all on the device,
    wall time of each call.  The pruned sweep kernel is timed by the library's
    CUDA events around every sweep launch."""
    out = []
    for item in spec.split(","):
        if not item:
            continue
        name, K = item.split(":")
        K = int(K)
        coords, _ = inputs.config_instance(name)
        n = len(coords)
        with tsp2opt.TSP2Opt(coords) as g:
            g.mf_tour()  # warm-up: MF workspace, candidate lists, kernels
            g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
            g.local_search_current(max_iters=2)
            g.set_option(tsp2opt.OPT_NEIGHBOURS, 0)
            t0 = time.perf_counter()
            m = g.mf_tour()
            t1 = time.perf_counter()
            g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
            r = g.local_search_current()
            t2 = time.perf_counter()
            g.set_option(tsp2opt.OPT_NEIGHBOURS, 0)
            f = g.local_search_current()
            t3 = time.perf_counter()
            # the pruned sweep's kernel time: a second, profiled run (events between the
            # kernels cost launch overlap, so the timed run above records none)
            g.set_option(tsp2opt.OPT_NEIGHBOURS, K)
            g.mf_tour()
            g.profile(True)
            g.local_search_current()
            sweep_ms, sweeps = g.profile_read()
            g.profile(False)
        entry = {"config": name, "n": n, "K": K, "start": "mf", "mf_seconds": t1 - t0, "mf_length": m["length"],
                 "pruned_seconds": t2 - t1, "pruned_iterations": r["iterations"], "pruned_length": r["length"],
                 "pruned_sweep_us_avg": 1e3 * sweep_ms / max(1, sweeps), "pruned_sweeps": sweeps,
                 "candidates_per_sweep": 2 * K * n,
                 "polish_seconds": t3 - t2, "polish_iterations": f["iterations"], "length": f["length"],
                 "seconds": t3 - t0}
        if with_oracle and n <= 20000:  # the oracle's MF tour is O(n^2 log n): the small configs only
            import oracle
            mt = oracle.mf_tour(coords)
            o0 = time.perf_counter()
            o = oracle.pruned_local_search(coords, mt, K)
            o1 = time.perf_counter()
            entry["cpu_oracle"] = {"seconds": o1 - o0, "iterations": o["iterations"], "length": o["length"],
                                   "matches_gpu": bool(o["iterations"] == r["iterations"] and o["length"] == r["length"]),
                                   "cores": oracle.num_threads(), "kind": "oracle",
                                   "sample": "the whole pruned local search from the oracle's own MF tour"}
        out.append(entry)
    return out


def time_25opt(tsp2opt, spec, with_oracle=True):
    """Best-improvement 2.5-opt (TSP2OPT_OPT_NODE_INSERTION; SURVEY §8(f) NEXT-4,
    L26 §VII "2.5-opt"; reading R19) from the Multiple Fragment start, wall time
    of the MF tour and of the local search (device-resident, as the `mf` entries
    of time_to_local_minimum); the 2.5-opt sweep kernel is timed by the
    library's CUDA events."""
    out = []
    for name in spec.split(","):
        if not name:
            continue
        coords, _ = inputs.config_instance(name)
        n = len(coords)
        with tsp2opt.TSP2Opt(coords) as g:
            g.set_option(tsp2opt.OPT_NODE_INSERTION, 1)
            g.mf_tour()  # warm-up
            g.local_search_current(max_iters=2)
            t0 = time.perf_counter()
            m = g.mf_tour()
            t1 = time.perf_counter()
            r = g.local_search_current()
            t2 = time.perf_counter()
            g.mf_tour()  # a second, profiled run for the sweep's kernel time
            g.profile(True)
            g.local_search_current()
            sweep_ms, sweeps = g.profile_read()
            g.profile(False)
        entry = {"config": name, "n": n, "start": "mf", "moves": "2-opt + node insertion", "seconds": t2 - t0,
                 "mf_seconds": t1 - t0, "ls_seconds": t2 - t1, "mf_length": m["length"],
                 "iterations": r["iterations"], "length": r["length"],
                 "sweep_us_avg": 1e3 * sweep_ms / max(1, sweeps), "sweeps": sweeps}
        if with_oracle and n <= 20000:
            import oracle
            mt = oracle.mf_tour(coords)
            reps = 10
            o0 = time.perf_counter()
            for _ in range(reps):
                oracle.best_move25(coords, mt)
            per = (time.perf_counter() - o0) / reps
            entry["cpu_oracle"] = {"sweep_seconds": per, "est_ls_seconds": per * (r["iterations"] + 1),
                                   "cores": oracle.num_threads(), "kind": "oracle",
                                   "sample": f"{reps} oracle 2.5-opt sweeps of the MF tour; the local search "
                                             "estimate is per-sweep time x (moves + 1)"}
        out.append(entry)
    return out


def time_oropt(tsp2opt, spec, with_oracle=True):
    """Best-improvement Or-opt (tsp2opt_oropt_local_search; SURVEY §8(f) NEXT-4
    "2.5-opt/Or-opt variants"; reading R21), `cfg` (random start) or
    `cfg:hilbert` entries: wall time of the stateless C-ABI call, host tour in
    and out, with the oracle's per-sweep time on the start tour beside it."""
    out = []
    for item in spec.split(","):
        if not item:
            continue
        name, _, tk = item.partition(":")
        coords, tour = inputs.config_instance(name, tk or "random")
        n = len(coords)
        tsp2opt.oropt_local_search(coords, tour, max_iters=2)  # warm-up
        t0 = time.perf_counter()
        r = tsp2opt.oropt_local_search(coords, tour)
        sec = time.perf_counter() - t0
        cells = n * (n - 1) // 2
        entry = {"config": name, "n": n, "start": tk or "random", "moves": "2-opt + Or-opt segments of 1..3 cities",
                 "seconds": sec, "iterations": r["iterations"], "length": r["length"],
                 "s_per_iteration": sec / (r["iterations"] + 1),
                 "pairs_covered_per_s": cells * (r["iterations"] + 1) / sec, "moves_per_pair": 13}
        if with_oracle and n <= 20000:
            import oracle
            reps = 3 if n > 5000 else 10
            o0 = time.perf_counter()
            for _ in range(reps):
                oracle.best_move_or(coords, tour)
            per = (time.perf_counter() - o0) / reps
            entry["cpu_oracle"] = {"sweep_seconds": per, "est_ls_seconds": per * (r["iterations"] + 1),
                                   "cores": oracle.num_threads(), "kind": "oracle",
                                   "sample": f"{reps} oracle Or-opt sweeps of the start tour; the local search "
                                             "estimate is per-sweep time x (moves + 1)"}
        out.append(entry)
    return out


def time_first(tsp2opt, spec):
    """First-improvement 2-opt (TSP2OPT_OPT_FIRST_IMPROVEMENT; SURVEY §8(f) NEXT-4;
    reading R20) to the local minimum, `cfg` (random start) or `cfg:mf` entries,
    wall time of tsp2opt_local_search (as time_to_local_minimum)."""
    out = []
    for item in spec.split(","):
        if not item:
            continue
        name, _, tk = item.partition(":")
        coords, tour = inputs.config_instance(name, "random")
        n = len(coords)
        with tsp2opt.TSP2Opt(coords) as g:
            if tk == "mf":
                tour = g.mf_tour()["tour"]
            g.set_option(tsp2opt.OPT_FIRST_IMPROVEMENT, 1)
            g.local_search(tour, max_iters=2)  # warm-up
            t0 = time.perf_counter()
            r = g.local_search(tour)
            dt = time.perf_counter() - t0
        out.append({"config": name, "n": n, "start": tk or "random", "rule": "first improvement", "seconds": dt,
                    "iterations": r["iterations"], "length": r["length"]})
    return out


def time_ils(tsp2opt, spec):
    """Iterated Local Search (Algorithm 1) throughput: `cfg:iterations` entries."""
    out = []
    for item in spec.split(","):
        name, _, iters = item.partition(":")
        iters = int(iters or 50)
        coords, tour = inputs.config_instance(name)
        with tsp2opt.TSP2Opt(coords) as g:
            g.ils(tour, 1, 7)  # warm-up
            t0 = time.perf_counter()
            r = g.ils(tour, iters, 2013)
            dt = time.perf_counter() - t0
        out.append({"config": name, "n": len(tour), "ils_iterations": iters, "seconds": dt,
                    "ils_iterations_per_s": iters / dt, "first_local_min": int(r["lengths"][0]),
                    "best_length": r["length"], "seed": 2013})
    return out


def time_batch(tsp2opt, spec, with_oracle=True):
    """Batched small-instance local search: `n:batch`
    entries; B independent uniform instances (seeds 1..B, random starts) solved
    to their local minima, one CTA each.  Device-resident (CUDA events around
    tsp2opt_batch_local_search_async) and end to end through the host API."""
    import torch

    out = []
    for item in spec.split(","):
        n, _, B = item.partition(":")
        n, B = int(n), int(B or 4736)
        cs = np.stack([inputs.make_coords("uniform", n, 1 + b) for b in range(B)]).astype(np.int32)
        ts = np.stack([inputs.random_tour(n, 1 + b) for b in range(B)]).astype(np.int32)
        dc, d0 = torch.from_numpy(cs).cuda(), torch.from_numpy(ts).cuda()
        dl = torch.zeros(B, dtype=torch.int64, device="cuda")
        di = torch.zeros(B, dtype=torch.int64, device="cuda")
        st = torch.cuda.current_stream()
        dev = []
        for rep in range(4):
            dt_ = d0.clone()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            tsp2opt.batch_local_search_async(dc.data_ptr(), n, B, dt_.data_ptr(), dl.data_ptr(), di.data_ptr(),
                                             stream=st.cuda_stream)
            e1.record()
            torch.cuda.synchronize()
            if rep:
                dev.append(e0.elapsed_time(e1) * 1e-3)
        dev_s = float(np.median(dev))
        moves = int(di.sum())
        tsp2opt.batch_local_search(cs[:2], ts[:2])  # warm-up of the host entry
        host = []
        for _ in range(3):  # median of 3 host-API runs
            t0 = time.perf_counter()
            r = tsp2opt.batch_local_search(cs, ts)
            host.append(time.perf_counter() - t0)
        host_s = float(np.median(host))
        ok = bool((r["lengths"] == dl.cpu().numpy()).all())
        item_out = {"n": n, "instances": B, "coords": "uniform seeds 1..B", "start": "random",
                    "device_s": dev_s, "instances_per_s": B / dev_s,
                    "pairs_per_s": (moves + B) * n * (n - 1) / 2 / dev_s, "mean_moves": moves / B,
                    "e2e_s": host_s, "e2e_instances_per_s": B / host_s, "e2e_h2d_bytes": int(cs.nbytes + ts.nbytes),
                    "e2e_d2h_bytes": int(ts.nbytes + 16 * B), "e2e_matches_device": ok, "gpu_launches": 1}
        if with_oracle:
            import oracle

            k, t1 = 0, time.perf_counter()
            while k < B and time.perf_counter() - t1 < 3.0:
                oracle.local_search(cs[k], ts[k])
                k += 1
            osec = time.perf_counter() - t1
            item_out["cpu_oracle"] = {"instances_per_s": k / osec, "sample": f"{k} instances one after another",
                                      "cores": oracle.num_threads()}
        out.append(item_out)
    return out


def time_batch_ils(tsp2opt, spec, with_oracle=True):
    """Batched Iterated Local Search (Algorithm 1):
    `cfg:replicas:steps` entries; multi-start on ONE instance of config cfg
    (replica b: random start tour seed 1000+b, perturbation seed 2013+b), one
    CTA per replica.  Device-resident (CUDA events around
    tsp2opt_batch_ils_async) and end to end through the host API."""
    import torch

    out = []
    for item in spec.split(","):
        name, R, T = item.split(":")
        R, T = int(R), int(T)
        c, _ = inputs.config_instance(name)
        n = len(c)
        cs = np.repeat(np.asarray(c, dtype=np.int32)[None], R, axis=0)
        ts = np.stack([inputs.make_tour("random", c, 1000 + b) for b in range(R)]).astype(np.int32)
        seeds = np.arange(2013, 2013 + R, dtype=np.uint64)
        dc, d0 = torch.from_numpy(cs).cuda(), torch.from_numpy(ts).cuda()
        ds = torch.from_numpy(seeds.view(np.int64)).cuda()
        dl = torch.zeros(R, dtype=torch.int64, device="cuda")
        st = torch.cuda.current_stream()
        dev = []
        for rep in range(3):
            dt_ = d0.clone()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            tsp2opt.batch_ils_async(dc.data_ptr(), n, R, dt_.data_ptr(), T, ds.data_ptr(), dl.data_ptr(),
                                    stream=st.cuda_stream)
            e1.record()
            torch.cuda.synchronize()
            if rep:
                dev.append(e0.elapsed_time(e1) * 1e-3)
        dev_s = float(np.median(dev))
        tsp2opt.batch_ils(cs[:2], ts[:2], 1, seeds[:2], history=False)  # warm-up of the host entry
        host = []
        for _ in range(3):  # median of 3 host-API runs
            t0 = time.perf_counter()
            r = tsp2opt.batch_ils(cs, ts, T, seeds, history=False)
            host.append(time.perf_counter() - t0)
        host_s = float(np.median(host))
        L = dl.cpu().numpy()
        item_out = {"config": name, "n": n, "replicas": R, "ils_steps": T, "device_s": dev_s,
                    "ils_steps_per_s": R * T / dev_s, "best_length": int(L.min()), "mean_length": float(L.mean()),
                    "e2e_s": host_s, "e2e_ils_steps_per_s": R * T / host_s,
                    "e2e_h2d_bytes": int(cs.nbytes + ts.nbytes + seeds.nbytes), "e2e_d2h_bytes": int(ts.nbytes + 8 * R),
                    "e2e_matches_device": bool((r["lengths"] == L).all()), "gpu_launches": 1}
        if with_oracle:
            import oracle

            k, t1 = 0, time.perf_counter()
            steps = max(1, T // 10)
            while k < R and time.perf_counter() - t1 < 3.0:
                oracle.ils(c, ts[k], steps, int(seeds[k]))
                k += 1
            osec = time.perf_counter() - t1
            item_out["cpu_oracle"] = {"ils_steps_per_s": k * steps / osec,
                                      "sample": f"{k} replicas x {steps} ILS steps one after another (each "
                                                f"includes its first local search)", "cores": oracle.num_threads()}
        out.append(item_out)
    return out


# ----------------------------------------------------------------------------- oracle timing
def cpu_baseline(args, coords, tour, total_pairs):
    import oracle

    t0 = time.perf_counter()
    sweeps = 0
    while True:
        oracle.best_move(coords, tour)
        sweeps += 1
        if time.perf_counter() - t0 > args.cpu_seconds or sweeps >= 3:
            break
    dt = time.perf_counter() - t0
    return {"value": sweeps * total_pairs / dt, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"{sweeps} full sweep(s) of the same workload (best_move over C(n,2) pairs), "
                      f"{dt:.1f} s, plain C oracle, OpenMP", "seconds": dt}


def run_reference(args):
    """--impl reference: the oracle (plain C, host cores) on our arm's config/metric."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle

    cfg = inputs.CONFIGS[args.config]
    n = cfg["n"]
    coords, tour = inputs.config_instance(args.config, args.tour)
    total_pairs = n * (n - 1) // 2
    oracle.build()
    for _ in range(min(args.warmup, 1)):
        oracle.best_move(coords, tour)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        i, j, d = oracle.best_move(coords, tour)
        t2 = oracle.apply(tour, i, j) if d < 0 else tour  # noqa: F841  (apply is part of the step)
        times.append(time.perf_counter() - t0)
        if sum(times) > args.ref_seconds:
            break
    k = len(times)
    value = total_pairs * k / sum(times)
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": max(world, args.gpus), "steps": k,
            "warmup": args.warmup,
            "ms_per_step": 1e3 * sum(times) / k, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int64", "data": "synthetic", "impl": "reference",
            "config": {"workload": f"{args.config} n={n} {cfg['coords']} coords, {args.tour} tour; one step = "
                                   "oracle best_move (C(n,2) pairs) + apply", "n": n},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
                             "sample": f"{k} step(s) of the workload (capped at {args.ref_seconds:.0f} s)"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def launch_ranks(n: int) -> int:
    import socket

    try:
        import torch

        have = torch.cuda.device_count()
    except Exception:  # pragma: no cover
        have = 0
    if have < n and "--exchange=p2p" not in sys.argv and "p2p" not in sys.argv:
        print(json.dumps({"metric": METRIC, "error": f"--gpus {n} but {have} CUDA device(s) visible"}), flush=True)
        return 2
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5")
    ap.add_argument("--tour", default="random", choices=["random", "hilbert"])
    ap.add_argument("--ls-config", default="C1,C2,C3,C4:hilbert,C5:hilbert,C2:mf,C3:mf,C4:mf,C5:mf", help="configs timed to a local minimum (rank 0, N=1)")
    ap.add_argument("--sharded-config", default="C4:hilbert,C5:hilbert,C4:mf,C5:mf",
                    help="time to local minimum on the sharded handle, N > 1 (every rank)")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "p2p"],
                    help="sharded exchange for N > 1; p2p also lets ranks share a GPU (a code-path check)")
    ap.add_argument("--balance-config", default="C4,C5", help="per-shard sweep times of the LPT split, N = 1")
    ap.add_argument("--ils-config", default="C1:200,C2:50", help="Iterated Local Search runs cfg:iterations")
    ap.add_argument("--pruned-config", default="C3:8,C4:8,C5:8,C5:16", help="pruned 2-opt from MF, cfg:K")
    ap.add_argument("--or25-config", default="C3,C4,C5", help="2.5-opt local search from MF, configs")
    ap.add_argument("--oropt-config", default="C1,C2,C3:hilbert", help="Or-opt local search, cfg[:hilbert]")
    ap.add_argument("--first-config", default="C1,C2,C3:mf,C4:mf,C5:mf", help="first-improvement local search")
    ap.add_argument("--batch-config", default="100:4736,1002:592", help="batched local search n:instances")
    ap.add_argument("--batch-ils-config", default="C1:4736:100", help="batched ILS cfg:replicas:steps")
    ap.add_argument("--no-ls", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--ref-seconds", type=float, default=120.0)
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        args.warmup = 3
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        # `bench.py --gpus N` without an external launcher: start the N ranks here
        # (one process per GPU, rendezvous on 127.0.0.1), exactly as torchrun would.
        raise SystemExit(launch_ranks(args.gpus))
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
