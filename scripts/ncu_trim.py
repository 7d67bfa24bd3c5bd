"""Trim an ncu --page source --csv export to the hottest SASS lines (by warp
stall samples) so that it fits in gpurun_out; usage: ncu_trim.py in.csv out.csv N"""
import csv
import sys

src, dst, n = sys.argv[1], sys.argv[2], int(sys.argv[3])
rows = []
hdr = None
with open(src, newline="") as f:
    for r in csv.reader(f):
        if hdr is None:
            if any("Source" in c for c in r) and any("Sampling" in c for c in r):
                hdr = r
            continue
        if len(r) == len(hdr):
            rows.append(r)
key = [i for i, c in enumerate(hdr) if "Warp Stall Sampling (All" in c]
k = key[0] if key else -1


def num(x):
    try:
        return float(x.replace(",", ""))
    except Exception:
        return 0.0


tot = sum(num(r[k]) for r in rows) if k >= 0 else 0
rows.sort(key=lambda r: -num(r[k]) if k >= 0 else 0)
with open(dst, "w", newline="") as f:
    w = csv.writer(f)
    w.writerow(["total_samples", tot, "lines", len(rows)])
    w.writerow(hdr)
    for r in rows[:n]:
        w.writerow(r)
