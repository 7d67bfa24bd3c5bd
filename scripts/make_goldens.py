"""Full-size parity goldens (SURVEY.md Sec. 8(c) "Parity at scale"): per-regex
match counts and the two position digests of the CPU oracle over a whole
BASELINE.json workload, written to tests/golden/full_<config>.tsv.

Only oracle/ computes the values (plain Thompson NFA + lazy DFA, oracle.c);
gen/ builds the seeded patterns and input.  Each file is keyed by the sha256
of the pattern list and of the input bytes, so a test can check that it
compares against the workload it regenerates.

Usage: python scripts/make_goldens.py snort [dotstar clamav multi1g] [--threads N]
"""
import hashlib
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402

# config -> (patterns, input, description); the bench workloads (bench.WORKLOADS)
# rebuilt here without importing bench (no product code on this path)
CFG = {
    "snort": (lambda: gen.snort_patterns(1000, 2)[0], lambda: gen.snort_input(256 << 20, seed=2),
              "snort-like 1k regexes x 256 MiB"),
    "clamav": (lambda: gen.clamav_brill_patterns(1000, 3)[0], lambda: gen.text_input(1 << 30, seed=3),
               "clamav/brill-like 2k regexes x 1 GiB"),
    "dotstar": (lambda: gen.dotstar_protomata_patterns(1000, 4)[0], lambda: gen.dotstar_input(1 << 30, seed=4),
                "dotstar/protomata-like 2k regexes x 1 GiB"),
    # config 5: all 10k regexes over a 64 MiB sample of the 8 GiB multi input
    # (the first 16 MiB of each of its four 2 GiB family parts, concatenated)
    # config 5 as the GPU tests build it in seconds: the 64 MiB multi stream
    # (four 16 MiB family parts, gen.multi_input(64 MiB)); the 8 GiB test
    # tiles it (tests/test_gpu_config5.py)
    "multi64": (lambda: gen.multi_patterns(2500), lambda: gen.multi_input(64 << 20, seed=5),
                "multi 10k regexes x 64 MiB (gen.multi_input(64 MiB, seed 5): four 16 MiB family parts)"),
    "multi64m": (lambda: gen.multi_patterns(2500), lambda: multi_sample(),
                 "multi 10k regexes x 64 MiB sample (first 16 MiB of each 2 GiB part of the 8 GiB input)"),
}


def multi_sample(each: int = 16 << 20) -> np.ndarray:
    return np.concatenate([gen.multi_input(8 << 30, seed=5, part=i)[:each] for i in range(4)])


def pattern_sha(pats) -> str:
    h = hashlib.sha256()
    for p in pats:
        h.update(len(p).to_bytes(8, "little"))
        h.update(p)
    return h.hexdigest()


def input_sha(data: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(data).data).hexdigest()


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    threads = os.cpu_count()
    if "--threads" in sys.argv:
        threads = int(sys.argv[sys.argv.index("--threads") + 1])
        args = [a for a in args if a != str(threads)]
    for name in args or ["snort"]:
        pb, ib, desc = CFG[name]
        pats = pb()
        data = ib()
        t = time.time()
        r = oracle.run_set(pats, data, threads=threads)
        dt = time.time() - t
        path = os.path.join(ROOT, "tests", "golden", f"full_{name}.tsv")
        with open(path, "w") as f:
            f.write(f"# {desc}: oracle (oracle/oracle.c, Thompson NFA + lazy DFA) counts and position digests\n")
            f.write(f"# written by scripts/make_goldens.py ({dt:.0f} s on {threads} threads)\n")
            f.write(f"patterns_sha256\t{pattern_sha(pats)}\n")
            f.write(f"input_sha256\t{input_sha(data)}\n")
            f.write(f"input_bytes\t{data.size}\n")
            f.write(f"n_regex\t{len(pats)}\n")
            for i in range(len(pats)):
                f.write(f"{i}\t{int(r['counts'][i])}\t{int(r['digests'][i, 0])}\t{int(r['digests'][i, 1])}\n")
        print(f"{name}: {len(pats)} regexes x {data.size} B in {dt:.0f} s -> {path}", flush=True)


if __name__ == "__main__":
    main()
