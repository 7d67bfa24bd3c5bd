"""The cross-regex literal prefilter (DESIGN.md
"Prefilter").

CPU tier: the factor chosen for each regex is a set of literal k-grams of
which one occurs inside every match (property (i) of DESIGN.md "Prefilter"),
checked by brute force with Python's ``re`` over all substrings of short
texts -- an oracle independent of the compiler.

GPU tier: with the prefilter on, the CUDA path stays bit-exact against the
CPU oracle, including factors planted across 1 KiB prefilter blocks and
window frames, state-carrying tails that outlive their factor by many
windows, and the Snort-like set.
"""
import re

import numpy as np
import pytest

import gen
import oracle
import paper_conf_micro_ge0025_b200 as rx


def _windows(toks):
    """factor tokens "vvmm..vvmm@ae" -> [(values, masks, ae)]"""
    out = []
    for tok in toks:
        body, ae = tok.split("@")
        vals = bytes(int(body[i:i + 2], 16) for i in range(0, len(body), 4))
        msks = bytes(int(body[i + 2:i + 4], 16) for i in range(0, len(body), 4))
        out.append((vals, msks, int(ae.split("/")[0])))
    return out


def factors(prog):
    """regex index -> (first windows or None, output windows or None, delta)
    from rx_program_info ("regex i: factor first W.. ; out W.. ; delta=D")."""
    out = {}
    for line in prog.info.splitlines():
        m = re.match(r"regex (\d+): factor first (.*) ; out (.*) ; delta=(\d+)", line)
        if not m:
            continue
        first = None if m.group(2).strip() == "none" else _windows(m.group(2).split())
        outw = None if m.group(3).strip() == "none" else _windows(m.group(3).split())
        out[int(m.group(1))] = (first, outw, int(m.group(4)))
    return out


def _occurrences(text, win):
    """anchor-end positions e of the masked window (the window's bytes are
    text[e - ae : e - ae + len]) lying wholly inside text"""
    vals, msks, ae = win
    n = len(vals)
    hits = []
    for st in range(0, len(text) - n + 1):
        if all((text[st + j] & msks[j]) == vals[j] for j in range(n)):
            hits.append((st, st + ae))
    return hits


HAND = [rb"abcd.*xyz", rb"(?:ab)+cdef", rb"wxyz[0-9]+q", rb"x(?:yz)*w", rb"(foo|ba[rz])", rb"q[^\n]*zz",
        rb"ab[cd]{2}e", rb"(?:kk|ll)mmnn", rb"[ab]{3}c+", rb"hello(?:,? world)?!", rb"a.{0,5}bcd",
        rb"[a-z]+wxyz", rb"abc(?:de)*", rb"q[0-9]{2}(mn|kl)rs", rb"(?:xy|zw)+qq"]


PLANTS = [b"abcdqqxyz", b"ababcdef", b"wxyz12q", b"xyzyzw", b"foo", b"bar", b"baz", b"q\nzz", b"qzz", b"abdce",
          b"kkmmnn", b"llmmnn", b"hello, world!", b"hello!", b"a12bcd", b"abcdede", b"q12mnrs", b"q34klrs",
          b"xyzwqq", b"zwxyqq", b"aabccc", b"kwxyz"]


def test_factor_occurs_in_every_match_bruteforce():
    # first factors: one lies inside every match (property (i)); output
    # factors: one lies inside every match with its anchor end at most delta
    # bytes before the match end (mode B) -- Python's re over all substrings
    rng = np.random.default_rng(5)
    pats = list(HAND)
    while len(pats) < 70:
        p = gen.fuzz_pattern(rng)
        if len(p) <= 20:
            pats.append(p)
    prog = rx.Program(pats, flags=rx.RX_F_MODEB)  # output factors exist only with mode B allowed
    fac = factors(prog)
    assert sum(v[0] is not None for v in fac.values()) >= 10
    assert sum(v[1] is not None for v in fac.values()) >= 10
    alphabet = b"abcdefkl mnqrswxyz0123!,\n"
    checked = {"first": 0, "out": 0}
    for trial in range(40):
        n = int(rng.integers(8, 40))
        if trial % 2:
            text = bytearray(gen.fuzz_text(rng, n))
        else:
            text = bytearray(alphabet[i] for i in rng.integers(0, len(alphabet), size=n))
        for _ in range(2):
            pl = PLANTS[int(rng.integers(0, len(PLANTS)))]
            at = int(rng.integers(0, max(1, n - len(pl))))
            text[at:at + len(pl)] = pl
        text = bytes(text)
        n = len(text)
        for i, p in enumerate(pats):
            first, outw, delta = fac[i]
            if first is None and outw is None:
                continue
            occ_f = [(st, len(w[0])) for w in (first or []) for (st, _) in _occurrences(text, w)]
            occ_o = [(st, e, len(w[0])) for w in (outw or []) for (st, e) in _occurrences(text, w)]
            cre = re.compile(p)
            for s in range(n):
                for e in range(s + 1, n + 1):
                    if not cre.fullmatch(text, s, e):
                        continue
                    if first is not None:
                        checked["first"] += 1
                        assert any(s <= st and st + ln <= e for (st, ln) in occ_f), (p, text[s:e], first)
                    if outw is not None:
                        checked["out"] += 1
                        assert any(s <= st and st + ln <= e and e - 1 - ae <= delta for (st, ae, ln) in occ_o), (
                            p, text[s:e], outw, delta)
    assert checked["first"] > 50 and checked["out"] > 50, checked


def test_factor_windows_are_long_and_exact():
    # extension windows: the whole fixed-offset literal prefix (<= 16 bytes),
    # alternations of words branch, classes of one bit stay compared
    prog = rx.Program([rb"HTTP/1\.union.+<script>", rb"GET(admin|root)xyz", rb"Cookie:[^\x00]*619ajavascript:",
                       rb"[Ss]elect\s+from"], flags=rx.RX_F_MODEB)
    fac = factors(prog)
    (f0, o0, _), (f1, _, _), (f2, o2, d2), (f3, _, _) = fac[0], fac[1], fac[2], fac[3]
    assert f0 is not None and bytes(v for v, m in zip(f0[0][0], f0[0][1]) if m == 0xff) == b"HTTP/1.union"
    assert o0 is not None and bytes(v for v, m in zip(o0[0][0], o0[0][1]) if m == 0xff) == b"<script>"
    assert sorted(bytes(w[0]) for w in f1) == [b"GETadminxyz", b"GETrootxyz"]
    assert bytes(f2[0][0]) == b"Cookie:" and bytes(o2[0][0]) == b"619ajavascript:" and d2 <= 15
    assert f3[0][1][0] == 0xdf and f3[0][0][1:6] == b"elect"   # [Ss] compared up to bit 5


def test_stateful_factor_precedes_first_unbounded_repetition():
    # property (ii): first factors are taken before the first unbounded
    # repetition; output factors from the suffix after the last one
    prog = rx.Program([rb"(?:ab)+cdef", rb"xyzw[0-9]+qrst", rb"abcd.*wxyz", rb"abcd[a-z]+"], flags=rx.RX_F_MODEB)
    fac = factors(prog)
    assert fac[0][0] is None                           # nothing mandatory before (ab)+
    assert bytes(fac[1][0][0][0]) == b"xyzw"           # not "qrst"
    assert bytes(fac[2][0][0][0]) == b"abcd"           # not "wxyz"
    assert bytes(fac[2][1][0][0]) == b"wxyz"           # output factor: the suffix
    assert fac[3][1] is None                           # ends in a class-plus: no output factor


gpu = pytest.mark.gpu


def _gpu_counts(prog, data, dense=False):
    import torch
    buf = torch.frombuffer(bytearray(data), dtype=torch.uint8).cuda() if data else torch.zeros(
        0, dtype=torch.uint8, device="cuda")
    out = prog.match(buf, dense=dense)
    torch.cuda.synchronize()
    r = {"counts": out["counts"].cpu().numpy().view(np.uint64), "digests": out["digests"].cpu().numpy().view(
        np.uint64), "status": int(out["status"].cpu()[0])}
    if dense:
        r["dense"] = out["dense"].cpu().numpy().view(np.uint32)[:, : (len(data) + 31) // 32]
    return r


def _plant_edges(rng, n, plants):
    alphabet = np.frombuffer(b"abcdefghijklmnopqrstuvwxyz0123456789 \n", dtype=np.uint8)
    buf = bytearray(alphabet[rng.integers(0, alphabet.size, size=n)].tobytes())
    spots = []
    for b in range(1024, n - 64, 1024):
        spots += [b - 3, b - 2, b - 1, b, b + 1]
    for w in range(2048 - 96, n - 64, 1984):
        spots += [w - 40, w - 1, w, w + 5]
    for at in spots:
        s = plants[int(rng.integers(0, len(plants)))]
        at = min(max(at, 0), n - len(s))
        buf[at:at + len(s)] = s
    return bytes(buf)


@gpu
def test_prefilter_edges_bit_exact():
    pats = list(HAND)
    plants = [b"abcd", b"abcdqqxyz", b"ababcdef", b"wxyz123q", b"xyzyzw", b"foo", b"bar", b"q" + b"y" * 3000 + b"zz",
              b"abdde", b"kkmmnn", b"hello, world!", b"a12bcd"]
    rng = np.random.default_rng(11)
    prog = rx.Program(pats)
    for n in (1, 777, 4096, 70001, 300000):
        data = _plant_edges(rng, n, plants)[:n]
        g = _gpu_counts(prog, data, dense=True)
        o = oracle.run_set(pats, data, dense=True)
        assert g["status"] == 0
        assert np.array_equal(g["counts"], o["counts"]), (n, g["counts"], o["counts"])
        assert np.array_equal(g["digests"], o["digests"])
        assert np.array_equal(g["dense"], o["dense"][:, : g["dense"].shape[1]])


@gpu
def test_prefilter_long_state_outlives_factor():
    # the factor "abcd" occurs once; the .* state then crosses ~100 windows
    pats = [rb"abcd.*xyz", rb"wxyz[0-9]+q", rb"abcd[^\x00]*\x00"]
    data = b"zz" * 1000 + b"abcd" + b"k" * 200000 + b"xyz" + b"wxyz" + b"7" * 150000 + b"q" + b"\x00"
    prog = rx.Program(pats)
    g = _gpu_counts(prog, data, dense=True)
    o = oracle.run_set(pats, data, dense=True)
    assert np.array_equal(g["counts"], o["counts"]) and np.array_equal(g["digests"], o["digests"])
    assert np.array_equal(g["dense"], o["dense"][:, : g["dense"].shape[1]])
    assert int(g["counts"].sum()) >= 3


@gpu
@pytest.mark.parametrize("n", [(2 << 20) + 777])
def test_snort_like_prefilter_vs_oracle(n):
    pats = gen.snort_patterns(1000, 2)[0]
    data = bytes(gen.snort_input(n, seed=2))
    prog = rx.Program(pats)
    assert "prefilter: on" in prog.info
    g = _gpu_counts(prog, data)
    o = oracle.run_set(pats, data)
    assert g["status"] == 0
    bad = np.nonzero(g["counts"] != o["counts"])[0]
    assert bad.size == 0, [(pats[i], int(g["counts"][i]), int(o["counts"][i])) for i in bad[:5]]
    assert np.array_equal(g["digests"], o["digests"])
    assert int(o["counts"].sum()) > 0


def _modeb_input(rng, n, hot, rare, kill=b"\x00", kill_every=50000):
    """text with a hot first factor every ~300 bytes, rare output factors
    planted near 1 KiB-block and window edges, kill bytes now and then"""
    alphabet = np.frombuffer(b"abcdefghijklmnopqrstuvwxyz0123456789 /=&.-", dtype=np.uint8)
    buf = bytearray(alphabet[rng.integers(0, alphabet.size, size=n)].tobytes())
    for at in range(int(rng.integers(0, 300)), n - 64, 300):
        buf[at:at + len(hot)] = hot
    spots = [int(x) for x in rng.integers(0, n - 64, size=12)] + [4093, 4095, 8190, 16383, 65535, 131070]
    for at in spots:
        if at + len(rare) < n:
            buf[at:at + len(rare)] = rare
    for at in range(kill_every // 2, n, kill_every):
        buf[at:at + len(kill)] = kill
    return bytes(buf)


@gpu
def test_mode_b_walk_back_bit_exact(capfd):
    # hot first factors ("Cookie:", "HTTP/1.") with rare output factors: the
    # clusters run output-gated (mode B) and reconstruct their incoming state
    # by walking back -- across long [^\x00]* carries, while-loop frontiers,
    # segment boundaries and up to the stream start
    pats = [rb"Cookie:[^\x00]*619ajavascript:", rb"HTTP/1\.(?:%[0-9a-f]{2})*DpPXrWa(?:iJ4/)*",
            rb"Cookie:[a-z]+=qz7Kx", rb"HTTP/1\.[^\r\n]*q9Zz", rb"zz[0-9]+", rb"abc"]
    rng = np.random.default_rng(3)
    prog = rx.Program(pats, flags=rx.RX_F_STATS | rx.RX_F_MODEB)
    plants = [b"619ajavascript:", b"%2f%3aDpPXrWaiJ4/iJ4/", b"DpPXrWa", b"abc=qz7Kx", b"q9Zz"]
    for n in (5000, 200000, (3 << 20) + 123):
        a = _modeb_input(rng, n, b"Cookie:", plants[0])
        b = _modeb_input(rng, n, b"HTTP/1.", plants[int(rng.integers(1, len(plants)))], kill=b"\r\n")
        # alternate 3 KiB pieces of the two texts
        data = b"".join((a if (i // 3072) % 2 else b)[i:i + 3072] for i in range(0, n, 3072))[:n]
        data = data[: n // 3] + b"Cookie:abc=qz7KxHTTP/1.%2fDpPXrWaiJ4/" + data[n // 3:]
        g = _gpu_counts(prog, data, dense=True)
        o = oracle.run_set(pats, data, dense=True)
        assert g["status"] == 0
        assert np.array_equal(g["counts"], o["counts"]), (n, g["counts"], o["counts"])
        assert np.array_equal(g["digests"], o["digests"])
        assert np.array_equal(g["dense"], o["dense"][:, : g["dense"].shape[1]])
    err = capfd.readouterr().err
    assert "modeB_members=" in err and re.search(r"modeB_members=[1-9]", err), err[-2000:]
    assert re.search(r"walkbacks=[1-9]", err), err[-2000:]


@gpu
def test_mode_b_off_equals_on():
    # mode B (RX_F_MODEB, opt-in) gives the same result on the Snort-like set
    pats = gen.snort_patterns(300, 2)[0]
    data = bytes(gen.snort_input((1 << 20) + 5, seed=7))
    a = _gpu_counts(rx.Program(pats, flags=rx.RX_F_MODEB), data)
    b = _gpu_counts(rx.Program(pats), data)
    assert np.array_equal(a["counts"], b["counts"]) and np.array_equal(a["digests"], b["digests"])
