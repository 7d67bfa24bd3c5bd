"""Step time with and without per-kernel profiling events, and the host time
of one rx_match call (launch path), on the bench workload."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_micro_ge0025_b200 as rx  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "snort"
pats, data, n, name = bench.load_workload(cfg)
prog = rx.Program(pats, **bench.PROGRAM_OPTS.get(cfg, {}))
d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
out = prog.alloc_outputs(d.numel(), d.device, dense=False, digests=False)
s = torch.cuda.current_stream()
for _ in range(3):
    prog.match(d, out=out, stream=s)
torch.cuda.synchronize()


def steps(k):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t = time.perf_counter()
    e0.record(s)
    for _ in range(k):
        prog.match(d, out=out, stream=s)
    host = (time.perf_counter() - t) / k
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / k, host * 1e3


print("profiling off: device ms/step %.3f, host ms/call %.3f" % steps(10))
prog.set_profiling(True)
prog.kernel_times(reset=True)
print("profiling on : device ms/step %.3f, host ms/call %.3f" % steps(10))
print(prog.kernel_times(reset=True))
prog.set_profiling(False)
