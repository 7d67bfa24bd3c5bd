"""One hot group of the Snort-like set as its own program (ncu source-level
profile of its pass 1 at a manageable code size).  Usage:
  python scripts/hot_group_profile.py <group id> [steps]"""
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_micro_ge0025_b200 as rx  # noqa: E402

gid = int(sys.argv[1]) if len(sys.argv) > 1 else 4
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
pats, data, n, name = bench.load_workload("snort")
full = rx.Program(pats, **bench.PROGRAM_OPTS["snort"])
m = re.search(r"^group %d: .* members=([\d,]+)" % gid, full.info, re.M)
ids = [int(x) for x in m.group(1).split(",")]
sub = [pats[i] for i in ids]
prog = rx.Program(sub, **bench.PROGRAM_OPTS["snort"])
print("group", gid, "regexes", len(sub), "groups", prog.n_groups, flush=True)
d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
out = prog.alloc_outputs(d.numel(), d.device, dense=False, digests=False)
prog.set_profiling(True)
for _ in range(steps):
    prog.match(d, out=out)
torch.cuda.synchronize()
print(prog.kernel_times(reset=True), "matches", int(out["counts"].sum()), flush=True)
