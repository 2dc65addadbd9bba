"""Aggregate an ncu source page (--page source --csv --print-source cuda,sass) by CUDA source line:
warp-stall samples and executed warp instructions per line, top N."""
import csv
import sys


def main(path, top=40):
    rows = list(csv.reader(open(path)))
    fname, agg, tot = "?", {}, 0.0
    hdr = None
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < 6 or r[0] in ("", "Function Name"):
            continue
        try:
            s = float(r[4])
            ins = float(r[7])
        except ValueError:
            continue
        k = (fname, int(r[0]))
        a = agg.setdefault(k, [0.0, 0.0, r[1][:90]])
        a[0] += s
        a[1] += ins
        tot += s
    print(f"# {path}: stall samples by source line (total {tot:.0f})")
    for (f, ln), (s, ins, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
        print(f"{100 * s / max(tot, 1):6.2f}% {ins:12.0f} inst  {f}:{ln}  {src.strip()}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)
