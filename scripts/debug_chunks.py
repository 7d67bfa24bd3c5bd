"""Single-process check of the chunk protocol on the test_gpu_multiproc workload:
end state of chunk 0, rematch of chunk 1, totals vs one rx_match."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_micro_ge0025_b200 as rx  # noqa: E402
from test_gpu_multiproc import _workload  # noqa: E402

pats, data = _workload()
prog = rx.Program(pats)
dev = torch.device("cuda", 0)
n = len(data)
cut = n // 2
d = torch.from_numpy(data).to(dev)
whole = prog.match(d)
torch.cuda.synchronize()
wc = whole["counts"].cpu().numpy().view(np.uint64)
lb, la = prog.lookback, prog.lookahead
print("lookback", lb, "lookahead", la, "boundary_bytes", prog.boundary_bytes, "whole total", int(wc.sum()))
st0 = prog.zero_state(dev) if hasattr(prog, "zero_state") else torch.zeros(max(prog.boundary_bytes // 4, 1), dtype=torch.int32, device=dev)
buf0 = d[: cut + la]
o0 = prog.match_chunk(buf0, cut, 0, la, 0, state_in=None, state_out=st0)
torch.cuda.synchronize()
print("chunk0 state nonzero words", int((st0 != 0).sum()), "of", st0.numel())
buf1 = d[cut - lb:]
zero = torch.zeros_like(st0)
st1 = torch.zeros_like(st0)
o1 = prog.match_chunk(buf1, n - cut, lb, 0, cut, state_in=zero, state_out=st1)
torch.cuda.synchronize()
c0 = o0["counts"].cpu().numpy().view(np.uint64)
c1 = o1["counts"].cpu().numpy().view(np.uint64)
print("speculative total", int(c0.sum() + c1.sum()), "diff regexes", np.nonzero(c0 + c1 != wc)[0][:10])
prog.rematch_chunk(buf1, n - cut, lb, 0, cut, zero, st0.clone(), st1, o1)
torch.cuda.synchronize()
c1 = o1["counts"].cpu().numpy().view(np.uint64)
print("after rematch total", int(c0.sum() + c1.sum()), "diff regexes", np.nonzero(c0 + c1 != wc)[0][:10])
