"""Accounting of the sparse pass 1 (rx_options.flags |= RX_F_STATS): window
visits, active windows, prefilter member hits, mode-B walk-backs, per group.
Usage: python scripts/stats_run.py [config] [length_mib] [--modeb]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))
import numpy as np  # noqa: E402

import bench  # noqa: E402
import paper_conf_micro_ge0025_b200 as rx  # noqa: E402

args = [a for a in sys.argv[1:] if not a.startswith("--")]
cfg = args[0] if args else "snort"
mib = int(args[1]) if len(args) > 1 else 0
pats, data, n, name = bench.load_workload(cfg, (mib << 20) if mib else None)
t = time.time()
flags = rx.RX_F_STATS | (rx.RX_F_MODEB if "--modeb" in sys.argv else 0)
prog = rx.Program(pats, flags=flags, **bench.PROGRAM_OPTS.get(cfg, {}))
print(f"compiled {len(pats)} regexes, {prog.n_groups} groups in {time.time() - t:.1f} s", flush=True)
if os.environ.get("RX_INFO_OUT"):
    open(os.environ["RX_INFO_OUT"], "w").write(prog.info)
try:
    import torch
    if torch.cuda.is_available():
        d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
        out = prog.alloc_outputs(data.size, d.device, dense=False, digests=False)
        prog.match(d, out=out)
        torch.cuda.synchronize()
        print("total matches:", int(out["counts"].sum()))
except Exception as e:  # noqa: BLE001
    print("no GPU run:", e)
