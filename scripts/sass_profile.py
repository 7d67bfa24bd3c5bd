"""Summaries of an `ncu --page source --csv --print-source sass` export
(gzip): opcode mix and the hottest address ranges.  usage: sass_profile.py f.csv.gz"""
import collections
import csv
import gzip
import io
import sys

rows = list(csv.reader(io.TextIOWrapper(gzip.open(sys.argv[1]))))
hdr = rows[1]
ie, ss, src = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source")
data = [r for r in rows[2:] if len(r) == len(hdr) and r[ie].isdigit()]
tot = sum(int(r[ie]) for r in data)
ts = sum(int(r[ss]) for r in data) or 1
print("instructions", tot, "samples", ts, "lines", len(data))
op, ops = collections.Counter(), collections.Counter()
for r in data:
    o = r[src].strip().split()
    if not o:
        continue
    k = (o[1] if o[0].startswith("@") else o[0]).split(".")[0]
    op[k] += int(r[ie])
    ops[k] += int(r[ss])
for k, v in op.most_common(22):
    print(f"{k:10s} {v / tot * 100:5.1f}% inst {ops[k] / ts * 100:5.1f}% samples")
W = int(sys.argv[2]) if len(sys.argv) > 2 else 64
blk = []
for i in range(0, len(data), W):
    b = data[i:i + W]
    blk.append((sum(int(r[ss]) for r in b) / ts * 100, sum(int(r[ie]) for r in b) / tot * 100, i,
                b[0][src].strip()[:60]))
print("hottest blocks of", W, "lines (samples %, inst %, line, first instruction)")
for x in sorted(blk, reverse=True)[:12]:
    print(f"  {x[0]:5.1f} {x[1]:5.1f} {x[2]:6d} {x[3]}")
