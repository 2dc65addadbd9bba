"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel: count, total, share."""
import csv
import sys
from collections import defaultdict


def main(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    hdr = rows[0]
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            k = d["Kernel Name"].split("(")[0]
            agg[k][0] += 1
            agg[k][1] += float(d["Metric Value"]) * (1e-3 if d["Metric Unit"] == "ns" else 1.0)
    # every kernel of libtsp2opt.so; the rest (PyTorch / NCCL / CUB helpers) is reported as not ours
    foreign = ("at::", "nccl", "cub::", "cutlass", "triton", "elementwise", "vectorized", "reduce_kernel", "CatArray")
    ours = {k: v for k, v in agg.items() if not any(f in k for f in foreign)}
    tot_ours = sum(v[1] for v in ours.values())
    print(f"# {path}: per-kernel device time (cold-cache, serialised; compare shares)")
    print(f"{'launches':>8} {'total_us':>12} {'avg_us':>10} {'share_of_ours':>13}  kernel")
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        share = f"{100 * v[1] / tot_ours:12.2f}%" if k in ours else "    (not ours)"
        print(f"{v[0]:8d} {v[1]:12.1f} {v[1] / v[0]:10.1f} {share}  {k}")


if __name__ == "__main__":
    main(sys.argv[1])
