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


def factors(prog):
    """regex index -> list of factor byte strings (None: always runs)."""
    out = {}
    for line in prog.info.splitlines():
        m = re.match(r"regex (\d+): factor (.*)", line)
        if not m:
            continue
        i = int(m.group(1))
        if m.group(2).startswith("none"):
            out[i] = None
            continue
        grams = []
        for tok in m.group(2).split("grams=")[1].strip(",").split(","):
            h, k = tok.split("/")
            g, k = int(h, 16), int(k)
            grams.append(bytes((g >> (8 * (4 - k + j))) & 255 for j in range(k)))
        out[i] = grams
    return out


HAND = [rb"abcd.*xyz", rb"(?:ab)+cdef", rb"wxyz[0-9]+q", rb"x(?:yz)*w", rb"(foo|ba[rz])", rb"q[^\n]*zz",
        rb"ab[cd]{2}e", rb"(?:kk|ll)mmnn", rb"[ab]{3}c+", rb"hello(?:,? world)?!", rb"a.{0,5}bcd"]


def test_factor_occurs_in_every_match_bruteforce():
    rng = np.random.default_rng(5)
    pats = list(HAND)
    while len(pats) < 60:
        p = gen.fuzz_pattern(rng)
        if len(p) <= 20:
            pats.append(p)
    prog = rx.Program(pats)
    fac = factors(prog)
    assert any(v is not None for v in fac.values())
    alphabet = b"abcdefkl mnqrwxyz0123!,\n"
    for _ in range(30):
        n = int(rng.integers(5, 40))
        text = bytes(alphabet[i] for i in rng.integers(0, len(alphabet), size=n))
        for i, p in enumerate(pats):
            grams = fac[i]
            if grams is None:
                continue
            cre = re.compile(p)
            for s in range(n):
                for e in range(s + 1, n + 1):
                    if cre.fullmatch(text, s, e):
                        sub = text[s:e]
                        assert any(g in sub for g in grams), (p, sub, grams)


def test_stateful_factor_precedes_first_unbounded_repetition():
    # property (ii): the factor is taken before the first unbounded repetition
    prog = rx.Program([rb"(?:ab)+cdef", rb"xyzw[0-9]+qrst", rb"abcd.*wxyz"])
    fac = factors(prog)
    assert fac[0] is None                      # nothing mandatory before (ab)+
    assert all(g in b"xyzw" for g in fac[1])   # not "qrst"
    assert all(g in b"abcd" for g in fac[2])   # not "wxyz"


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
