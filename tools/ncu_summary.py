"""Summarise an ncu --set full report (raw page) into the handful of numbers DESIGN.md / profiles/ cite."""
import csv
import io
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "sm_clock"),
    ("smsp__inst_executed.sum", "warp_inst_total"),
    ("sm__inst_executed.avg.per_cycle_active", "ipc_per_sm (max 4)"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_active_pct"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "pipe_alu_pct"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "pipe_fma_pct"),
    ("sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active", "pipe_fmaheavy_cycles_pct"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "pipe_xu_pct"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "pipe_lsu_pct"),
    ("sm__warps_active.avg.per_cycle_active", "warps_active_per_sm"),
    ("launch__registers_per_thread", "registers"),
    ("launch__occupancy_limit_registers", "occ_limit_regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
]
STALLS = "smsp__average_warps_issue_stalled_"


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for vals in rows[2:]:
        d = dict(zip(hdr, vals))
        u = dict(zip(hdr, units))
        print(f"# {d.get('Kernel Name', '?')[:90]}")
        for k, name in KEYS:
            if k in d:
                print(f"{name:28s} {d[k]} {u.get(k, '')}")
        st = sorted(((float(v), k[len(STALLS):].replace("_per_issue_active.ratio", ""))
                     for k, v in d.items() if k.startswith(STALLS) and k.endswith("_per_issue_active.ratio")
                     and v not in ("", "n/a")), reverse=True)
        print("stalls per issue (top):", ", ".join(f"{n}={v:.2f}" for v, n in st[:8]))


if __name__ == "__main__":
    for p in sys.argv[1:]:
        main(p)
