"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Each pin is chosen so that a plausible mistake in the oracle (a dropped
epsilon edge, an off-by-one in the match-end position, an anchored start, a
wrong class, a bad R{n,m} expansion, a stale DFA cache) fails at least one:

* values PAPER.md prints for its worked examples (tests/golden/*.tsv, cited);
* brute force: S[i] = OR_s re.fullmatch(p, text[s:i+1]) with Python's `re`
  (a backtracking library routine; bytes mode, default flags: '.' excludes
  '\\n', [^x] includes it -- the readings of DESIGN.md), on a random grammar;
* closed forms (a single class counts its bytes; literal sets = naive
  overlapping memmem; a* = the 'a' positions under non-empty semantics);
* invariants (ends(a|b) = ends(a) U ends(b); adding alternatives is monotone);
* the memoised DFA equals the plain NFA simulation;
* the digest equals an independent Python splitmix64.
"""
import ast
import os
import re

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def ends_of(pattern, data, **kw):
    return set(int(p) for p in oracle.Regex(pattern).run(data, positions=True, **kw)["positions"])


def brute_ends(pattern: bytes, data: bytes):
    rx = re.compile(pattern)
    out = set()
    for i in range(len(data)):
        for s in range(i + 1):
            if rx.fullmatch(data, s, i + 1):
                out.add(i)
                break
    return out


def _nested_repeat(pattern: bytes) -> bool:
    """True if a repeat (max > 1) contains another repeat: Python's backtracking
    `re` can take exponential time there, so such patterns get short texts."""
    from re import _parser as sp  # CPython's own regex parser (library routine)

    def walk(items, inside):
        for op, av in items:
            if op in (sp.MAX_REPEAT, sp.MIN_REPEAT):
                lo, hi, sub = av
                if inside and hi != 0:
                    return True
                if walk(sub, inside or hi is sp.MAXREPEAT or hi > 1):
                    return True
            elif op == sp.SUBPATTERN:
                if walk(av[-1], inside):
                    return True
            elif op == sp.BRANCH:
                if any(walk(b, inside) for b in av[1]):
                    return True
        return False

    return walk(sp.parse(pattern), False)


def _golden_rows(name):
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            yield line.rstrip("\n").split("\t")


@pytest.mark.parametrize("row", list(_golden_rows("paper_examples.tsv")), ids=lambda r: r[0] + ":" + r[1])
def test_paper_worked_examples(row):
    pat, data, exp, cite = row
    data = ast.literal_eval(data)
    expected = set() if exp == "-" else {int(x) for x in exp.split(",")}
    assert ends_of(pat, data) == expected, cite
    assert ends_of(pat, data, use_cache=False) == expected, cite


def test_fig3_final_stream_matches_golden():
    rows = dict((r[0], r[1]) for r in _golden_rows("paper_streams.tsv"))
    s9 = {int(x) for x in rows["S9"].split(",")}
    assert ends_of(b"(abc)|d", b"abcdabce") == s9


def test_basis_formula_for_a():
    # 'a' = not b0 & b1 & b2 & not b3 & not b4 & not b5 & not b6 & b7 (b0 = MSB)
    data = bytes(range(256))
    want = {c for c in range(256)
            if (not (c >> 7) & 1) and (c >> 6) & 1 and (c >> 5) & 1 and not (c >> 4) & 1
            and not (c >> 3) & 1 and not (c >> 2) & 1 and not (c >> 1) & 1 and (c & 1)}
    assert want == {0x61}
    assert ends_of(b"a", data) == want


def test_brute_force_random_grammar():
    rng = np.random.default_rng(12345)
    n_checked = 0
    for _ in range(260):
        p = gen.fuzz_pattern(rng)
        t = gen.fuzz_text(rng, int(rng.integers(1, 12 if _nested_repeat(p) else 40)))
        want = brute_ends(p, t)
        assert ends_of(p, t) == want, (p, t)
        assert ends_of(p, t, use_cache=False) == want, (p, t)
        n_checked += 1
    assert n_checked == 260


def test_brute_force_byte_alphabet():
    # full byte alphabet incl. 0x00, 0xFF and '\n': classes, dot, escapes
    rng = np.random.default_rng(7)
    pats = [rb".", rb"[^a]", rb"\x00+", rb"[\x80-\xff]{2}", rb"\d\s", rb"\w+", rb"\W", rb"\S\D",
            rb"[^\n]*\n", rb"\xff.", rb"[a\-z]", rb"[]a]", rb"\.\*", rb"(\x00|\n)(\x00|\n)"]
    for p in pats:
        t = bytes(rng.integers(0, 256, size=60, dtype=np.uint8)) + b"a-z]*.\n\x00\x00\n 1a_\t9"
        assert ends_of(p, t) == brute_ends(p, t), p


def test_dot_and_negated_class_newline_reading():
    data = b"a\nb"
    assert ends_of(b".", data) == {0, 2}          # '.' excludes '\n' (c4)
    assert ends_of(b"[^x]", data) == {0, 1, 2}    # negated class includes '\n' (c4)


def test_nonempty_semantics():
    data = b"baab"
    assert ends_of(b"a*", data) == {1, 2}    # c1: only non-empty matches
    assert ends_of(b"(a|)", data) == {1, 2}
    assert ends_of(b"", data) == set()
    assert ends_of(b"()*", data) == set()
    assert ends_of(b"x?", data) == set()


def test_single_class_closed_form():
    rng = np.random.default_rng(3)
    data = rng.integers(0, 256, size=5000, dtype=np.uint8).tobytes()
    digits = {i for i, c in enumerate(data) if 0x30 <= c <= 0x39}
    assert ends_of(rb"[0-9]", data) == digits
    assert ends_of(rb"\d", data) == digits
    nonnl = {i for i, c in enumerate(data) if c != 10}
    assert ends_of(rb".", data) == nonnl
    assert ends_of(rb"[^\n]+", data) == nonnl
    r = oracle.Regex(rb"[\x00-\xff]").run(data)
    assert r["count"] == len(data)


def test_literal_sets_vs_naive_memmem():
    rng = np.random.default_rng(11)
    data = bytes(rng.choice(np.frombuffer(b"abcab", dtype=np.uint8), size=4000))
    for lit in [b"a", b"ab", b"abc", b"aa", b"aaa", b"cab", b"bcabca", b"abcabcab"]:
        want = set()
        s = data.find(lit)
        while s >= 0:
            want.add(s + len(lit) - 1)
            s = data.find(lit, s + 1)  # overlapping
        assert ends_of(re.escape(lit), data) == want, lit


def test_union_invariant_and_monotonicity():
    rng = np.random.default_rng(99)
    for _ in range(60):
        a, b = gen.fuzz_pattern(rng), gen.fuzz_pattern(rng)
        t = gen.fuzz_text(rng, 300)
        ea, eb = ends_of(a, t), ends_of(b, t)
        eab = ends_of(b"(?:" + a + b")|(?:" + b + b")", t)
        assert eab == ea | eb
        assert ea <= eab and eb <= eab


def test_bounded_repetition_closed_form():
    # a{n,m} over runs of a: position i ends a match iff the run of 'a' ending at i has length >= n (n >= 1)
    data = b"baaaabaaaaaaabaab" * 5
    for n, m in [(1, 1), (2, 3), (3, 3), (0, 2), (4, 9), (2, 64)]:
        run = 0
        want = set()
        for i, c in enumerate(data):
            run = run + 1 if c == ord("a") else 0
            if run >= max(n, 1):
                want.add(i)
        assert ends_of(b"a{%d,%d}" % (n, m), data) == want, (n, m)


def test_cache_equals_nfa_with_flushes():
    rng = np.random.default_rng(5)
    for _ in range(40):
        p = gen.fuzz_pattern(rng, depth=3)
        t = gen.fuzz_text(rng, 3000)
        r0 = oracle.Regex(p).run(t, use_cache=False)
        r1 = oracle.Regex(p).run(t, use_cache=True, max_states=3)  # tiny cache: frequent flushes
        r2 = oracle.Regex(p).run(t, use_cache=True)
        for r in (r1, r2):
            assert r["count"] == r0["count"] and r["d1"] == r0["d1"] and r["d2"] == r0["d2"]
            assert np.array_equal(r["dense"], r0["dense"])


def _splitmix64(x):
    m = (1 << 64) - 1
    z = (x + 0x9E3779B97F4A7C15) & m
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & m
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & m
    return z ^ (z >> 31)


def test_digests_and_dense_consistency():
    data = gen.tiny_input()
    r = oracle.Regex(b"[0-9]+x").run(data, positions=True)
    pos = [int(p) for p in r["positions"]]
    m = (1 << 64) - 1
    assert r["d1"] == sum(_splitmix64(p) for p in pos) & m
    assert r["d2"] == sum(_splitmix64(p ^ 0x9E3779B97F4A7C15) for p in pos) & m
    dense = r["dense"]
    bits = [w * 32 + b for w in range(dense.size) for b in range(32) if (int(dense[w]) >> b) & 1]
    assert bits == pos and r["count"] == len(pos)
    assert oracle.splitmix64(12345) == _splitmix64(12345)


def test_run_set_equals_single_runs():
    pats = gen.tiny_patterns()
    data = gen.tiny_input()
    rs = oracle.run_set(pats, data, threads=3, dense=True)
    for i, p in enumerate(pats):
        r = oracle.Regex(p).run(data)
        assert rs["counts"][i] == r["count"]
        assert rs["digests"][i, 0] == r["d1"] and rs["digests"][i, 1] == r["d2"]
        assert np.array_equal(rs["dense"][i], r["dense"])


def test_tiny_long_chain_is_found():
    data = gen.tiny_input()
    chain_end = 20000 + 1 + 2 * 10000
    assert data[20000:20000 + 4] == b"abcb" and data[chain_end] == ord("d")
    assert chain_end in ends_of(b"a(bc)*d", data)


@pytest.mark.parametrize("pat,code", [(b"^a", 2), (b"a$", 2), (b"a**", 1), (b"*a", 1), (b"(a", 1),
                                      (b"a)", 1), (b"[a", 1), (b"a{3,1}", 1), (b"\\1", 2), (b"a*?", 2),
                                      (b"(?=a)", 2), (b"\\bx", 2), (b"a{2000}", 3), (b"\\q", 1)])
def test_rejected_constructs(pat, code):
    assert oracle.check(pat)[0] == code


@pytest.mark.parametrize("pat,want", [(b"abc", 3), (b"a{2,5}", 5), (b"(ab|c)+", -1), (b"a?|bcd", 3), (b"a*|bcd", -1),
                                      (b"x(ab){3}y?", 8), (b"[0-9]+x", -1), (b"(a?){4}", 4), (b"()*", 0),
                                      (b"a.{0,32}b", 34), (b"(foo|ba[rz])", 3)])
def test_max_len_closed_forms(pat, want):
    assert oracle.Regex(pat).max_len == want


def test_max_len_bounds_every_brute_force_match():
    # the longest match found by brute force (all starts, all ends) never
    # exceeds max_len, and reaches it on a text made of the longest member
    rng = np.random.default_rng(777)
    for _ in range(150):
        p = gen.fuzz_pattern(rng)
        ml = oracle.Regex(p).max_len
        t = gen.fuzz_text(rng, int(rng.integers(1, 12 if _nested_repeat(p) else 30)))
        rx = re.compile(p)
        longest = max([i + 1 - s for i in range(len(t)) for s in range(i + 1) if rx.fullmatch(t, s, i + 1)],
                      default=0)
        if ml >= 0:
            assert longest <= ml, (p, t, longest, ml)
