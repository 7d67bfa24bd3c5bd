"""Config 5 of BASELINE.json: the 10k-regex multi-pattern set (2,500 per
family: Snort-like, ClamAV-like, Brill-like, Dotstar/Protomata-like) -- the
program that needs several linked modules.

* every one of the 10,000 regexes over the 64 MiB multi stream
  (gen.multi_input(64 MiB): four 16 MiB family parts): per-regex counts and
  both position digests equal the CPU oracle's (tests/golden/full_multi64.tsv,
  written by scripts/make_goldens.py, which calls only oracle/);
* at 8 GiB: that stream tiled 128 times (positions beyond 2^32).  For every
  regex with a finite longest match M_r (oracle max_len) the count is exact
  by construction: a match ending in tile k >= 1 depends only on the tile
  and the M = max M_r bytes before it, which are the same for every k, so
      count = 128 c0 + 127 (c1 - c0_head)
  with c0 the golden count of one tile, c1 the oracle's count of matches
  ending in the first M bytes of a tile preceded by the previous tile's last
  M bytes, c0_head the same without them (both oracle runs on 2M bytes).
  The match list checks the rest: its size equals the sum of the counts, its
  per-regex histogram equals the counts, its positions reach past 2^32 and
  the digests recomputed from it equal the kernel's.
"""
import hashlib
import os

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden", "full_multi64.tsv")
_G = np.uint64(0x9E3779B97F4A7C15)


def _golden():
    hdr, rows = {}, []
    with open(GOLDEN) as f:
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


def _splitmix64(x):
    with np.errstate(over="ignore"):
        z = x + _G
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


@pytest.fixture(scope="module")
def workload():
    if not os.path.exists(GOLDEN):
        pytest.skip("tests/golden/full_multi64.tsv not generated")
    pats = gen.multi_patterns(2500)
    data = gen.multi_input(64 << 20, seed=5)
    hdr, c, d1, d2 = _golden()
    h = hashlib.sha256()
    for p in pats:
        h.update(len(p).to_bytes(8, "little"))
        h.update(p)
    assert hdr["patterns_sha256"] == h.hexdigest()
    assert hdr["input_sha256"] == hashlib.sha256(np.ascontiguousarray(data).data).hexdigest()
    return pats, np.ascontiguousarray(data), rx.Program(pats), c, d1, d2


def test_config5_every_regex_64mib_vs_golden(workload):
    pats, data, prog, g_c, g_d1, g_d2 = workload
    assert len(pats) == 10000
    d = torch.from_numpy(data).cuda()
    out = prog.match(d, digests=True)
    torch.cuda.synchronize()
    counts = out["counts"].cpu().numpy().view(np.uint64)
    dig = out["digests"].cpu().numpy().view(np.uint64)
    assert int(out["status"].cpu()[0]) == 0
    bad = np.nonzero((counts != g_c) | (dig[:, 0] != g_d1) | (dig[:, 1] != g_d2))[0]
    assert bad.size == 0, [(int(i), pats[i][:60], int(counts[i]), int(g_c[i])) for i in bad[:8]]
    assert int(g_c.sum()) > 0


def test_config5_8gib_tiled(workload):
    pats, data, prog, g_c, _, _ = workload
    tiles = 128
    T = data.size
    ml = np.array([oracle.Regex(p).max_len for p in pats])
    bounded = np.nonzero(ml >= 0)[0]
    M = int(ml[bounded].max())
    assert 0 < M < T
    sub = [pats[r] for r in bounded]
    seam = np.concatenate([data[T - M:], data[:M]])
    pos_seam = oracle.positions_set(sub, bytes(seam))
    pos_head = oracle.positions_set(sub, bytes(data[:M]))
    delta = np.array([np.count_nonzero(p >= M) for p in pos_seam], dtype=np.int64) - \
        np.array([p.size for p in pos_head], dtype=np.int64)
    want = tiles * g_c[bounded].astype(np.int64) + (tiles - 1) * delta

    dev = torch.device("cuda", 0)
    big = torch.from_numpy(data).to(dev).repeat(tiles)
    assert big.numel() == tiles * T and big.numel() > (1 << 32)
    # list room: unbounded regexes may match more in later tiles (carries)
    total = 2 * int(g_c.sum()) * tiles + 4 * int(np.abs(delta).sum()) * tiles + (16 << 20)
    out = prog.alloc_outputs(big.numel(), dev, dense=False, digests=True, match_cap=total)
    prog.match(big, out=out)
    torch.cuda.synchronize()
    del big
    counts = out["counts"].cpu().numpy().view(np.uint64)
    dig = out["digests"].cpu().numpy().view(np.uint64)
    assert int(out["status"].cpu()[0]) == 0
    got = counts[bounded].astype(np.int64)
    bad = np.nonzero(got != want)[0]
    assert bad.size == 0, [(int(bounded[i]), pats[bounded[i]][:60], int(got[i]), int(want[i])) for i in bad[:8]]
    reg, pos = prog.match_list(out)
    assert reg.size == int(counts.sum())
    assert np.array_equal(np.bincount(reg, minlength=len(pats)).astype(np.uint64), counts)
    assert int(pos.max()) >= (1 << 32) and int(pos.max()) < tiles * T
    with np.errstate(over="ignore"):
        d1 = np.zeros(len(pats), dtype=np.uint64)
        d2 = np.zeros(len(pats), dtype=np.uint64)
        np.add.at(d1, reg, _splitmix64(pos))
        np.add.at(d2, reg, _splitmix64(pos ^ _G))
    assert np.array_equal(d1, dig[:, 0]) and np.array_equal(d2, dig[:, 1])
