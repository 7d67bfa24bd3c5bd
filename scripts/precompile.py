"""Fill the in-tree cubin cache (.rxcache/) for the workload configs, so that
GPU runs (which ship the cache in the gpurun snapshot) do not spend box time
in NVRTC.  Usage: python scripts/precompile.py [snort clamav dotstar multi tiny]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))

import bench  # noqa: E402
import gen  # noqa: E402
import paper_conf_micro_ge0025_b200 as rx  # noqa: E402

SETS = {
    "tiny": lambda: gen.tiny_patterns(),
    "snort": lambda: gen.snort_patterns(1000, 2)[0],
    "clamav": lambda: gen.clamav_brill_patterns(1000, 3)[0],
    "dotstar": lambda: gen.dotstar_protomata_patterns(1000, 4)[0],
    "multi": lambda: gen.multi_patterns(2500),
}

for name in sys.argv[1:] or list(SETS):
    t = time.time()
    prog = rx.Program(SETS[name](), **bench.PROGRAM_OPTS.get(name, {}))  # the bench's launch configuration
    if name == "snort":
        rx.Program(SETS[name]())  # the default geometry too (tests)
    print(f"{name}: {prog.n_regex} regexes, {prog.n_groups} groups, {time.time() - t:.1f} s", flush=True)
