"""Seeded synthetic pattern sets and inputs for the five BASELINE.json configs.

Every generator is a pure function of its seed.  Recipes (DESIGN.md "Input
recipe"):

  tiny      4 regexes (abc, [0-9]+x, a(bc)*d, (foo|ba[rz])) over 64 KiB ASCII
  snort     ~1k Snort-like regexes over 256 MiB packet payloads
  clamav    1k ClamAV-like hex signatures + 1k Brill-like word rules, 1 GiB text
  dotstar   1k Dotstar-like + 1k PROSITE-like motifs, 1 GiB (long lines)
  multi     10k regexes (2.5k per family) over 8 GiB (4 x 2 GiB family inputs)

Pattern sizes follow PAPER.md Table 1: e.g. Snort length
mean 50.5 / SD 41.5 chars, Protomata 96.5 / 36.2, ClamAV
359.7 / 310.7, Brill 44.4 / 16.9.  Inputs are synthetic
(no datasets); the paper used 10^6-byte real inputs.
"""
from __future__ import annotations

import re

import numpy as np

TINY_PATTERNS = [b"abc", b"[0-9]+x", b"a(bc)*d", b"(foo|ba[rz])"]


def tiny_patterns():
    return list(TINY_PATTERNS)


def _printable(rng, n):
    return rng.integers(0x20, 0x7F, size=n, dtype=np.uint8)


def tiny_input(seed: int = 1, length: int = 65536, long_chain: int = 10000) -> bytes:
    """Config 1: 70% from 'abcdfoxrz0123456789', 30% printable, '\\n' p=1/64;
    planted abc x200, digits+x x100, a(bc)^k d (k in [0,64]) x100 plus one
    chain with k=long_chain (20,002 B > one 16,384-bit block of P:L503),
    foo/bar/baz x100; plants straddle 31/32, 1023/1024, 16383/16384 and the
    last byte."""
    rng = np.random.default_rng(seed)
    alpha = np.frombuffer(b"abcdfoxrz0123456789", dtype=np.uint8)
    buf = alpha[rng.integers(0, alpha.size, size=length)]
    pr = rng.random(length) < 0.3
    buf = np.where(pr, _printable(rng, length), buf).astype(np.uint8)
    buf[rng.random(length) < 1.0 / 64] = ord("\n")
    out = bytearray(buf.tobytes())

    def put(at, s):
        at = max(0, min(at, length - len(s)))
        out[at:at + len(s)] = s

    for _ in range(200):
        put(int(rng.integers(0, length)), b"abc")
    for _ in range(100):
        k = int(rng.integers(1, 12))
        put(int(rng.integers(0, length)), bytes(rng.integers(0x30, 0x3A, size=k, dtype=np.uint8)) + b"x")
    for _ in range(100):
        k = int(rng.integers(0, 65))
        put(int(rng.integers(0, length)), b"a" + b"bc" * k + b"d")
    for _ in range(100):
        put(int(rng.integers(0, length)), [b"foo", b"bar", b"baz"][int(rng.integers(0, 3))])
    # straddles: matches that end exactly across word / warp-window / 16K boundaries
    for b in (32, 1024, 16384):
        if b + 8 < length:
            put(b - 2, b"abc")                    # ends at b
            put(b - 1 - 3, b"a" + b"bc" * 1 + b"d")  # a(bc)d ending at b-1 +...
            put(b + 2, b"123x")
            put(b - 3 + 8, b"foo")
    # the long chain last among the interior plants, so that it stays intact
    if long_chain and length > 2 * long_chain + 4 + 20000:
        put(20000, b"a" + b"bc" * long_chain + b"d")
    # the last byte
    put(length - 3, b"baz")
    return bytes(out[:length])


# ---------------------------------------------------------------------------
# random-grammar fuzz (tests): patterns in the supported subset whose Python
# `re` (bytes) meaning is the paper's (dot excludes \n, [^x] includes it).
# ---------------------------------------------------------------------------
_FUZZ_ALPHA = b"abc"


def _fuzz_atom(rng, depth):
    r = rng.random()
    if depth > 0 and r < 0.22:
        return b"(" + _fuzz_alt(rng, depth - 1) + b")", True
    if r < 0.30:
        return b"(?:" + _fuzz_alt(rng, depth - 1 if depth > 0 else 0) + b")", True
    if r < 0.40:
        c = [b"[ab]", b"[^a]", b"[a-c]", b"[^\\n]", b"[bc\\n]", b"\\d", b"[^ab]"][int(rng.integers(0, 7))]
        return c, True
    if r < 0.46:
        return b".", True
    if r < 0.50:
        return b"\\n", True
    return bytes([_FUZZ_ALPHA[int(rng.integers(0, len(_FUZZ_ALPHA)))]]), True


def _fuzz_piece(rng, depth):
    atom, _ = _fuzz_atom(rng, depth)
    r = rng.random()
    if r < 0.12:
        return atom + b"*"
    if r < 0.20:
        return atom + b"+"
    if r < 0.27:
        return atom + b"?"
    if r < 0.33:
        n = int(rng.integers(0, 4))
        m = n + int(rng.integers(0, 3))
        return atom + (b"{%d}" % n if rng.random() < 0.3 else b"{%d,%d}" % (n, m))
    if r < 0.35:
        return atom + b"{%d,}" % int(rng.integers(0, 3))
    return atom


def _fuzz_cat(rng, depth):
    n = int(rng.integers(1, 4))
    return b"".join(_fuzz_piece(rng, depth) for _ in range(n))


def _fuzz_alt(rng, depth):
    parts = [_fuzz_cat(rng, depth)]
    while rng.random() < 0.25:
        parts.append(_fuzz_cat(rng, depth) if rng.random() < 0.9 else b"")
    return b"|".join(parts)


def fuzz_pattern(rng, depth: int = 2) -> bytes:
    """A random pattern over {a,b,c,\\n,digits} that Python's `re` accepts."""
    while True:
        p = _fuzz_alt(rng, depth)
        try:
            re.compile(p)
            return p
        except re.error:
            continue


def fuzz_text(rng, n: int) -> bytes:
    alpha = np.frombuffer(b"abcabcab\n01", dtype=np.uint8)
    return alpha[rng.integers(0, alpha.size, size=n)].tobytes()


CONFIGS = {}  # filled below: name -> dict(patterns=callable, input=callable, ...)


def make_config(name: str, **kw):
    """(patterns, input bytes-like numpy u8 array) for a named config."""
    cfg = CONFIGS[name]
    return cfg["patterns"](**{k: v for k, v in kw.items() if k in cfg.get("pattern_kw", ())}), \
        cfg["input"](**{k: v for k, v in kw.items() if k in cfg.get("input_kw", ())})


CONFIGS["tiny"] = {
    "patterns": lambda: tiny_patterns(),
    "input": lambda length=65536, seed=1: np.frombuffer(tiny_input(seed, length), dtype=np.uint8),
    "input_kw": ("length", "seed"),
    "len": 65536,
    "desc": "tiny: 4 regexes over 64 KiB synthetic ASCII (seed 1)",
}
