"""Fill the in-tree cubin cache for the programs the -m gpu tests build
beyond the bench configurations (so a GPU box does not spend test time in
NVRTC).  Usage: python scripts/precompile_tests.py"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))

import gen  # noqa: E402
import paper_conf_micro_ge0025_b200 as rx  # noqa: E402

jobs = [
    ("rebalance snort", lambda: rx.Program(gen.snort_patterns(1000, 2)[0], flags=rx.RX_F_REBALANCE)),
    ("rebalance clamav", lambda: rx.Program(gen.clamav_brill_patterns(1000, 3)[0], flags=rx.RX_F_REBALANCE)),
    ("rebalance dotstar", lambda: rx.Program(gen.dotstar_protomata_patterns(1000, 4)[0], flags=rx.RX_F_REBALANCE)),
    ("multiproc", lambda: rx.Program(gen.dotstar_protomata_patterns(1000, 4)[0][::8] + gen.tiny_patterns())),
    ("host", lambda: rx.Program(gen.tiny_patterns() + gen.dotstar_protomata_patterns(1000, 4)[0][::20])),
    ("batch", lambda: rx.Program(gen.snort_patterns(1000, 2)[0][::5])),
    ("modeb", lambda: rx.Program(gen.snort_patterns(300, 2)[0], flags=rx.RX_F_MODEB)),
    ("plain300", lambda: rx.Program(gen.snort_patterns(300, 2)[0])),
]
for name, fn in jobs:
    t = time.time()
    p = fn()
    print(f"{name}: {p.n_regex} regexes, {p.n_groups} groups, {time.time() - t:.1f} s", flush=True)
