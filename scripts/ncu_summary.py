"""Markdown summary of an ncu --set full capture (profiles/rNN_ncu_*.md).
usage: ncu_summary.py details.csv raw.csv out.md "title" """
import csv
import sys

det, raw, out, title = sys.argv[1:5]
WANT = ["Duration", "Elapsed Cycles", "SM Frequency", "Compute (SM) Throughput", "Executed Ipc Active",
        "Issue Slots Busy", "Executed Instructions", "Registers Per Thread", "Achieved Active Warps Per SM",
        "Warp Cycles Per Issued Instruction", "L2 Hit Rate", "L1/TEX Hit Rate", "DRAM Throughput", "Grid Size",
        "Block Size", "Dynamic Shared Memory Per Block", "Achieved Occupancy"]
RAW = ["dram__bytes_read.sum", "dram__bytes_write.sum", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
       "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]
launches = {}
with open(det, newline="") as f:
    rows = [r for r in csv.reader(f)]
hdr = next(r for r in rows if "Metric Name" in r)
ix = {c: i for i, c in enumerate(hdr)}
for r in rows[rows.index(hdr) + 1:]:
    if len(r) <= ix["Metric Value"]:
        continue
    k = (r[ix["ID"]], r[ix["Kernel Name"]].split("(")[0])
    d = launches.setdefault(k, {})
    name = r[ix["Metric Name"]]
    if name in WANT and name not in d:
        d[name] = f"{r[ix['Metric Value']]} {r[ix['Metric Unit']]}".strip()
rawv = []  # raw-page rows in launch order (the trimmed export has no ID column)
with open(raw, newline="") as f:
    rr = list(csv.reader(f))
h = rr[0]
for r in rr[2:]:
    if len(r) == len(h):
        rawv.append({m: (r[h.index(m)], rr[1][h.index(m)]) for m in RAW if m in h})
with open(out, "w") as f:
    f.write(f"# {title}\n\n")
    for j, ((i, name), d) in enumerate(sorted(launches.items(), key=lambda kv: int(kv[0][0]))):
        f.write(f"## launch {i}: `{name}`\n\n| metric | value |\n|---|---|\n")
        for m in WANT:
            if m in d:
                f.write(f"| {m} | {d[m]} |\n")
        for m, (v, u) in (rawv[j] if j < len(rawv) else {}).items():
            f.write(f"| {m} | {v} {u} |\n")
        f.write("\n")
print(open(out).read()[:3000])
