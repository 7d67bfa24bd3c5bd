"""GPU parity at BASELINE.json's full sizes, in the launch configuration
bench.py times (SURVEY.md Sec. 8(c) "Parity at scale").

The whole input is matched once through the C ABI exactly as bench.py does
(same input bytes, same program, same rx_match launch geometry), with the
compacted match list on.  The oracle cannot scan 256 MiB - 1 GiB with 1-2k
regexes in test time, so it checks what it can compute one by one:

* the prefix: a match ending at i depends only on bytes <= i, so the
  oracle's positions on input[0, P) equal the listed positions < P, for every
  regex (bit-exact);
* sampled windows: for each regex with a finite longest match M_r (oracle
  max_len), matches ending in [a, b) depend only on input[a - M, b) with
  M = max M_r, so the oracle on that slice gives them exactly -- including the
  window ending at the last byte of the stream;
* properties at any size: the list holds sum(counts) entries, its per-regex
  histogram equals the counts, and the position digests recomputed from it
  equal the kernel's digests.
"""
import os
import sys

import numpy as np
import pytest

import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
import bench  # noqa: E402  (the bench's own workload builders)

pytestmark = pytest.mark.gpu

_G = np.uint64(0x9E3779B97F4A7C15)


def _splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = x + _G
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def _full_run(config, cap):
    pats, data, nbytes, _ = bench.load_workload(config)
    prog = rx.Program(pats, **bench.PROGRAM_OPTS.get(config, {}))  # the bench's launch configuration
    dev = torch.device("cuda", 0)
    d_in = torch.from_numpy(np.ascontiguousarray(data)).to(dev)
    out = prog.alloc_outputs(nbytes, dev, dense=False, digests=True, match_cap=cap)
    prog.match(d_in, out=out, stream=torch.cuda.current_stream(dev))
    torch.cuda.synchronize()
    counts = out["counts"].cpu().numpy().view(np.uint64)
    digests = out["digests"].cpu().numpy().view(np.uint64)
    assert int(out["status"].cpu()[0]) == 0
    reg, pos = prog.match_list(out)
    del d_in, out
    torch.cuda.empty_cache()
    return pats, data, counts, digests, reg, pos


def _check(config, cap, prefix, windows, seed):
    pats, data, counts, digests, reg, pos = _full_run(config, cap)
    n, ln = len(pats), int(data.size)
    # properties at full size
    assert reg.size == int(counts.sum())
    assert np.array_equal(np.bincount(reg, minlength=n).astype(np.uint64), counts)
    assert pos.size == 0 or int(pos.max()) < ln
    with np.errstate(over="ignore"):
        d1 = np.zeros(n, dtype=np.uint64)
        d2 = np.zeros(n, dtype=np.uint64)
        np.add.at(d1, reg, _splitmix64(pos))
        np.add.at(d2, reg, _splitmix64(pos ^ _G))
    assert np.array_equal(d1, digests[:, 0]) and np.array_equal(d2, digests[:, 1])
    starts = np.searchsorted(reg, np.arange(n + 1))

    def listed(r, lo, hi):
        p = pos[starts[r]:starts[r + 1]]
        return p[(p >= lo) & (p < hi)]

    # exact prefix, every regex
    ref = oracle.positions_set(pats, data[:prefix])
    for r in range(n):
        assert np.array_equal(listed(r, 0, prefix), ref[r]), (r, pats[r][:60])
    # sampled windows (and the stream's last bytes), regexes with finite longest match
    ml = np.array([oracle.Regex(p).max_len for p in pats])
    bounded = np.nonzero(ml >= 0)[0]
    assert bounded.size > 0
    M = int(ml[bounded].max())
    rng = np.random.default_rng(seed)
    W = 1 << 16
    offs = sorted(set([ln - W] + [int(x) for x in rng.integers(prefix, ln - W, size=windows)]))
    sub = [pats[r] for r in bounded]
    for a in offs:
        lo = max(0, a - M)
        got = oracle.positions_set(sub, data[lo:a + W])
        for j, r in enumerate(bounded):
            want = got[j] + np.uint64(lo)
            want = want[want >= np.uint64(a)]
            assert np.array_equal(listed(r, a, a + W), want), (a, r, pats[r][:60])
    assert int(counts.sum()) > 0


def _golden(name):
    """tests/golden/full_<name>.tsv (scripts/make_goldens.py: the CPU oracle
    over the whole workload) -> (header dict, counts, d1, d2)"""
    hdr, rows = {}, []
    with open(os.path.join(ROOT, "tests", "golden", f"full_{name}.tsv")) as f:
        for line in f:
            if line.startswith("#"):
                continue
            parts = line.rstrip("\n").split("\t")
            if len(parts) == 2:
                hdr[parts[0]] = parts[1]
            else:
                rows.append([int(x) for x in parts])
    a = np.array(rows, dtype=np.uint64)
    return hdr, a[:, 1], a[:, 2], a[:, 3]


def _sha(pats, data):
    import hashlib
    h = hashlib.sha256()
    for p in pats:
        h.update(len(p).to_bytes(8, "little"))
        h.update(p)
    return h.hexdigest(), hashlib.sha256(np.ascontiguousarray(data).data).hexdigest()


@pytest.mark.parametrize("config", ["snort", "dotstar", "clamav"])
def test_full_size_every_regex_vs_golden(config):
    """Every regex of the config, over the WHOLE input, in the launch
    configuration bench.py times: per-regex counts and both position digests
    equal the CPU oracle's (tests/golden/full_<config>.tsv, written by
    scripts/make_goldens.py, which calls only oracle/)."""
    hdr, g_counts, g_d1, g_d2 = _golden(config)
    pats, data, nbytes, _ = bench.load_workload(config)
    ps, ds = _sha(pats, data)
    assert hdr["patterns_sha256"] == ps and hdr["input_sha256"] == ds, "golden is for another workload"
    prog = rx.Program(pats, **bench.PROGRAM_OPTS.get(config, {}))
    dev = torch.device("cuda", 0)
    d_in = torch.from_numpy(np.ascontiguousarray(data)).to(dev)
    out = prog.alloc_outputs(nbytes, dev, dense=False, digests=True)
    prog.match(d_in, out=out, stream=torch.cuda.current_stream(dev))
    torch.cuda.synchronize()
    counts = out["counts"].cpu().numpy().view(np.uint64)
    digests = out["digests"].cpu().numpy().view(np.uint64)
    assert int(out["status"].cpu()[0]) == 0
    bad = np.nonzero((counts != g_counts) | (digests[:, 0] != g_d1) | (digests[:, 1] != g_d2))[0]
    assert bad.size == 0, [(int(i), pats[i][:60], int(counts[i]), int(g_counts[i])) for i in bad[:8]]
    assert int(g_counts.sum()) > 0
    del d_in, out
    torch.cuda.empty_cache()


def test_snort_like_full_256mib_sampled():
    _check("snort", cap=64 << 20, prefix=6 << 20, windows=12, seed=21)


def test_dotstar_protomata_full_1gib_sampled():
    _check("dotstar", cap=16 << 20, prefix=9 << 20, windows=12, seed=41)
