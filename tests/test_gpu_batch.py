"""GPU parity of rx_match_batch: many independent
streams in one call.  Each stream must equal the oracle run on that stream
alone -- bit-exact counts, digests and dense match-end bits -- so no match or
carried state (MatchStar runs, while-loop frontiers) crosses a boundary.
Streams are ragged, include empty ones, and are cut inside long matches."""
import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

pytestmark = pytest.mark.gpu

PATS = gen.tiny_patterns() + [rb"abcd.*xyz", rb"q[^z]*z", rb"(ab|cd)+e", rb"a[a-z]*b"]


def _check_batch(pats, streams, offset_pad=0):
    prog = rx.Program(pats)
    data = b"".join(streams)
    offs = np.cumsum([0] + [len(s) for s in streams]).astype(np.uint64)
    buf = torch.zeros(len(data) + 64, dtype=torch.uint8, device="cuda")
    if data:
        buf[: len(data)] = torch.frombuffer(bytearray(data), dtype=torch.uint8).cuda()
    cap = 1 << 16
    out = prog.match_batch(buf[: len(data)], offs, dense=True, match_cap=cap)
    torch.cuda.synchronize()
    assert int(out["status"].cpu()[0]) == 0
    counts = out["counts"].cpu().numpy().view(np.uint64)
    digests = out["digests"].cpu().numpy().view(np.uint64)
    dense = out["dense"].cpu().numpy().view(np.uint32)
    reg, pos = rx.Program.match_list(out)
    total = 0
    for i, s in enumerate(streams):
        o = oracle.run_set(pats, s, dense=True)
        assert np.array_equal(counts[i], o["counts"]), (i, len(s))
        # digests hash positions relative to the batch buffer (include/rx.h)
        exp = [[0, 0] for _ in pats]
        for r, ends in enumerate(oracle.positions_set(pats, s)):
            for j in ends:
                q = int(offs[i]) + int(j)
                exp[r][0] = (exp[r][0] + oracle.splitmix64(q)) % (1 << 64)
                exp[r][1] = (exp[r][1] + oracle.splitmix64(q ^ 0x9E3779B97F4A7C15)) % (1 << 64)
        assert np.array_equal(digests[i], np.array(exp, dtype=np.uint64).reshape(-1, 2)), (i, len(s))
        w = (len(s) + 31) // 32
        for r in range(len(pats)):
            assert np.array_equal(dense[i, r, :w], o["dense"][r][:w]), (i, pats[r])
            assert not dense[i, r, w:].any()
            # list entries of this stream are exactly the oracle's ends + offset
            sel = (reg == r) & (pos >= offs[i]) & (pos < offs[i + 1])
            bits = np.unpackbits(o["dense"][r][:w].view(np.uint8), bitorder="little")[: len(s)]
            assert np.array_equal(pos[sel] - offs[i], np.nonzero(bits)[0].astype(np.uint64))
        total += int(o["counts"].sum())
    assert len(reg) == total


def test_batch_ragged_streams_match_oracle_per_stream():
    rng = np.random.default_rng(11)
    base = gen.tiny_input()
    cuts = sorted(set(int(x) for x in rng.integers(0, len(base), 23)) | {0, 5, 5, 37, 1024, 1025, len(base)})
    streams = [base[a:b] for a, b in zip(cuts[:-1], cuts[1:])] + [b"", b"abc", b"a" + b"bc" * 3000 + b"d"]
    _check_batch(PATS, streams)


def test_batch_state_does_not_cross_boundaries():
    # every match here would need bytes of two streams: none may be reported
    streams = [b"ab", b"c", b"a" + b"bc" * 700, b"d", b"abcd", b"xyz", b"q" + b"y" * 5000, b"z", b"fo", b"o"]
    _check_batch(PATS, streams)


def test_batch_empty():
    prog = rx.Program(PATS)
    buf = torch.zeros(16, dtype=torch.uint8, device="cuda")
    out = prog.match_batch(buf[:0], [0])
    assert out["counts"].shape == (0, len(PATS))
    out = prog.match_batch(buf[:0], [0, 0, 0])
    torch.cuda.synchronize()
    assert int(out["counts"].abs().sum()) == 0


def test_batch_rejects_decreasing_offsets():
    prog = rx.Program(PATS)
    buf = torch.zeros(64, dtype=torch.uint8, device="cuda")
    with pytest.raises(rx.RxError):
        prog.match_batch(buf, [0, 40, 30, 64])


def test_batch_many_packets_snort_like():
    # thousands of packet-sized streams (0-1460 B) of Snort-like payload in ONE
    # launch sequence, with a Snort-like pattern subset: per-stream counts and
    # digests equal the oracle run on each stream alone
    pats = gen.snort_patterns(1000, 2)[0][::5]
    data = bytes(gen.snort_input(3 << 20, seed=12))
    rng = np.random.default_rng(12)
    lens = rng.integers(0, 1461, size=3000)
    offs = np.concatenate([[0], np.cumsum(lens)]).astype(np.uint64)
    assert int(offs[-1]) <= len(data)
    prog = rx.Program(pats)
    buf = torch.frombuffer(bytearray(data[: int(offs[-1])]), dtype=torch.uint8).cuda()
    out = prog.match_batch(buf, offs)
    torch.cuda.synchronize()
    assert int(out["status"].cpu()[0]) == 0
    counts = out["counts"].cpu().numpy().view(np.uint64)
    digests = out["digests"].cpu().numpy().view(np.uint64)
    regs = [oracle.Regex(p) for p in pats]  # compiled once, run per stream
    nz = 0
    for i in range(len(lens)):
        s = data[int(offs[i]):int(offs[i + 1])]
        exp_c = np.zeros(len(pats), dtype=np.uint64)
        exp_d = np.zeros((len(pats), 2), dtype=np.uint64)
        for r, rg in enumerate(regs):
            res = rg.run(s, dense=False, positions=True)
            exp_c[r] = res["count"]
            for j in res["positions"]:
                q = int(offs[i]) + int(j)
                exp_d[r, 0] = (int(exp_d[r, 0]) + oracle.splitmix64(q)) % (1 << 64)
                exp_d[r, 1] = (int(exp_d[r, 1]) + oracle.splitmix64(q ^ 0x9E3779B97F4A7C15)) % (1 << 64)
        assert np.array_equal(counts[i], exp_c), i
        assert np.array_equal(digests[i], exp_d), i
        nz += int(exp_c.sum())
    assert nz > 0
