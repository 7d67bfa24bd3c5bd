"""Config 5 (10k regexes) over a 4 MiB prefix, outside pytest (native
backtrace with LD_PRELOAD=scripts/segv_trace.so)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_micro_ge0025_b200 as rx  # noqa: E402

pats = gen.multi_patterns(2500)
t = time.time()
prog = rx.Program(pats)
print(f"compiled {prog.n_regex} regexes {prog.n_groups} groups {time.time() - t:.1f}s", flush=True)
print(prog.info.splitlines()[:5], flush=True)
data = gen.multi_input(int(sys.argv[1]) if len(sys.argv) > 1 else 4 << 20, seed=5)
d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
print("matching", flush=True)
out = prog.match(d, digests=True)
torch.cuda.synchronize()
print("status", int(out["status"].cpu()[0]), "total", int(out["counts"].sum()), flush=True)
