"""From an `ncu --page raw --csv` export, the DRAM bytes (read + write) and
the executed warp / thread instructions per launch of each kernel, written as
profiles/ncu_traffic.json for bench.py's roofline `traffic` field and its
integer-pipe block.  usage: ncu_traffic.py raw.csv workload input_bytes out.json [source]"""
import csv
import json
import sys

raw, workload, nbytes, out = sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4]
rows = list(csv.reader(open(raw)))
hdr, units = rows[0], rows[1]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
ik = hdr.index("Kernel Name")
cols = [hdr.index("dram__bytes_read.sum"), hdr.index("dram__bytes_write.sum")]
it = hdr.index("gpu__time_duration.sum") if "gpu__time_duration.sum" in hdr else None
iw = hdr.index("smsp__inst_executed.sum") if "smsp__inst_executed.sum" in hdr else None
ith = hdr.index("sass__thread_inst_executed_per_opcode_category") \
    if "sass__thread_inst_executed_per_opcode_category" in hdr else None
src = sys.argv[5] if len(sys.argv) > 5 else raw
acc = {}
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    k = r[ik]
    b = sum(float(r[c].replace(",", "")) * scale.get(units[c], 1) for c in cols)
    t = float(r[it].replace(",", "")) if it is not None else 0.0
    e = acc.setdefault(k, [0.0, 0, 0.0, units[it] if it is not None else "", 0.0, 0.0])
    e[0] += b
    e[1] += 1
    e[2] += t
    e[4] += float(r[iw].replace(",", "")) if iw is not None else 0.0
    e[5] += float(r[ith].replace(",", "")) if ith is not None else 0.0
res = {workload: {k: {"dram_bytes_per_launch": v[0] / v[1], "launches": v[1], "input_bytes": nbytes,
                      "ncu_duration_per_launch": v[2] / v[1], "duration_unit": v[3],
                      "warp_inst_per_launch": v[4] / v[1], "thread_inst_per_launch": v[5] / v[1], "source": src}
                  for k, v in acc.items()}}
try:
    old = json.load(open(out))
except Exception:
    old = {}
old.update(res)
json.dump(old, open(out, "w"), indent=1)
print(json.dumps(res, indent=1))
