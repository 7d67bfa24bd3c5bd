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


# ---------------------------------------------------------------------------
# token-based pattern builder: every token renders as regex text and can
# sample a member string (for planting matches)
# ---------------------------------------------------------------------------
_SPECIAL = set(b".^$*+?()[]{}|\\")


def _lit_regex(bs: bytes) -> bytes:
    out = bytearray()
    for c in bs:
        if c in _SPECIAL:
            out += b"\\" + bytes([c])
        elif 0x20 <= c < 0x7F:
            out.append(c)
        else:
            out += b"\\x%02x" % c
    return bytes(out)


class _Tok:
    """regex text + a sampler of member strings."""

    def __init__(self, text: bytes, sampler):
        self.text = text
        self.sample = sampler


def _lit(bs: bytes) -> _Tok:
    return _Tok(_lit_regex(bs), lambda rng, bs=bs: bs)


_CLASSES = {
    rb"\d": bytes(range(0x30, 0x3A)),
    rb"\s": b" \t\r\n\f\v",
    rb"[^\r\n]": bytes(c for c in range(256) if c not in (10, 13)),
    rb"[A-Za-z0-9]": bytes(range(0x30, 0x3A)) + bytes(range(0x41, 0x5B)) + bytes(range(0x61, 0x7B)),
    rb"[a-z]": bytes(range(0x61, 0x7B)),
    rb"[0-9a-f]": bytes(range(0x30, 0x3A)) + bytes(range(0x61, 0x67)),
    rb".": bytes(c for c in range(256) if c != 10),
    rb"[^\x00]": bytes(range(1, 256)),
    rb"\w": bytes(range(0x30, 0x3A)) + bytes(range(0x41, 0x5B)) + bytes(range(0x61, 0x7B)) + b"_",
}


def _quantified(body_text: bytes, body_sample, lo: int, hi: int, qtext: bytes) -> _Tok:
    def s(rng, lo=lo, hi=hi):
        n = int(rng.integers(lo, (hi if hi >= 0 else lo + 4) + 1))
        return b"".join(body_sample(rng) for _ in range(n))
    return _Tok(body_text + qtext, s)


def _class_tok(rng, name=None, quant=True, max_m=64) -> _Tok:
    names = list(_CLASSES)
    name = name or names[int(rng.integers(0, len(names)))]
    members = _CLASSES[name]
    one = (lambda r, m=members: bytes([m[int(r.integers(0, len(m)))]]))
    if not quant:
        return _Tok(name, one)
    q = rng.random()
    if q < 0.30:
        return _quantified(name, one, 1, -1, b"+")
    if q < 0.55:
        return _quantified(name, one, 0, -1, b"*")
    if q < 0.65:
        return _quantified(name, one, 0, 1, b"?")
    n = int(rng.integers(0, 9))
    m = n + int(rng.integers(0, max(1, max_m - n)))
    m = min(m, max_m)
    if rng.random() < 0.3:
        return _quantified(name, one, n, n, b"{%d}" % n)
    return _quantified(name, one, n, m, b"{%d,%d}" % (n, m))


def _alt_tok(words) -> _Tok:
    text = b"(" + b"|".join(_lit_regex(w) for w in words) + b")"
    return _Tok(text, lambda rng, w=words: w[int(rng.integers(0, len(w)))])


_SNORT_WORDS = [b"GET", b"POST", b"HEAD", b"/cgi-bin/", b"cmd.exe", b"/etc/passwd", b"admin", b"login", b"SELECT",
                b"union", b"<script>", b".php", b"?id=", b"User-Agent:", b"Content-Length:", b"Host:", b"Cookie:",
                b"/bin/sh", b"wget ", b"eval(", b"base64_decode", b"%2e%2e%2f", b"../", b"\\x90\\x90", b"HTTP/1.",
                b"Authorization: Basic ", b"filename=", b"boundary=", b".exe", b"document.cookie", b"onload=",
                b"javascript:", b"/admin/", b"password=", b"username=", b"action=", b"Referer:", b"PUT", b"DELETE",
                b"/index.", b"xp_cmdshell", b"exec(", b"system(", b"Accept-Language:", b"Content-Type:"]
_SNORT_ALTS = [[b"GET", b"POST", b"HEAD"], [b"/", b"\\"], [b"admin", b"root", b"user"],
               [b"select", b"union", b"insert"], [b"http", b"https", b"ftp"], [b"%20", b"+", b" "]]
_WORD_ALPHA = b"abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789_-/.=&%"


def _snort_literal(rng) -> bytes:
    r = rng.random()
    if r < 0.45:
        w = _SNORT_WORDS[int(rng.integers(0, len(_SNORT_WORDS)))]
        return w.replace(b"\\x90", b"\x90")
    if r < 0.85:
        n = int(rng.integers(3, 13))
        return bytes(_WORD_ALPHA[int(i)] for i in rng.integers(0, len(_WORD_ALPHA), size=n))
    n = int(rng.integers(2, 7))  # binary signature bytes
    return bytes(rng.integers(0, 256, size=n, dtype=np.uint8))


def _group_star(rng) -> _Tok:
    """A non-CC star (lowered to a while loop, P:L147 / Listing 3)."""
    r = rng.random()
    if r < 0.4:
        sep = bytes([b"/.-_&;"[int(rng.integers(0, 6))]])
        body = _Tok(_lit_regex(sep) + rb"[a-z0-9]+", lambda g, s=sep: s + bytes(
            _WORD_ALPHA[:36][int(i)] for i in g.integers(0, 36, size=int(g.integers(1, 5)))))
    elif r < 0.7:
        body = _Tok(rb"%[0-9a-f]{2}", lambda g: b"%" + bytes(b"0123456789abcdef"[int(i)] for i in g.integers(0, 16, 2)))
    else:
        w = _snort_literal(rng)[:4] or b"ab"
        body = _Tok(_lit_regex(w), lambda g, w=w: w)
    q = b"*" if rng.random() < 0.6 else b"+"
    lo = 0 if q == b"*" else 1
    return _quantified(b"(?:" + body.text + b")", body.sample, lo, -1, q)


def _lognormal_len(rng, mean, sd, lo=4, hi=None):
    s2 = np.log(1 + (sd / mean) ** 2)
    mu = np.log(mean) - s2 / 2
    v = float(rng.lognormal(mu, np.sqrt(s2)))
    v = max(lo, v)
    if hi:
        v = min(v, hi)
    return int(round(v))


def snort_patterns(n: int = 1000, seed: int = 2):
    """Snort-like set (Table 1 Snort: 1,873 regexes, length mean 50.5, SD 41.5,
    P:L394; ~2.5 while loops per regex).  Returns (patterns, samplers)."""
    rng = np.random.default_rng(seed)
    pats, samplers = [], []
    for _ in range(n):
        target = _lognormal_len(rng, 50.5, 41.5, lo=6, hi=400)
        toks = [_lit(_snort_literal(rng))]
        size = len(toks[0].text)
        while size < target:
            r = rng.random()
            if r < 0.60:
                t = _lit(_snort_literal(rng))
            elif r < 0.80:
                t = _class_tok(rng)
            elif r < 0.85:
                t = _alt_tok(_SNORT_ALTS[int(rng.integers(0, len(_SNORT_ALTS)))])
            else:
                t = _group_star(rng)
            toks.append(t)
            size += len(t.text)
        pats.append(b"".join(t.text for t in toks))
        samplers.append(lambda g, toks=toks: b"".join(t.sample(g) for t in toks))
    return pats, samplers


def _text_pool(rng, n: int, vocab) -> np.ndarray:
    words = rng.integers(0, len(vocab), size=n // 4)
    out = b"".join(vocab[int(i)] for i in words)
    return np.frombuffer(out[:n], dtype=np.uint8)


_HTTP_VOCAB = [b"GET ", b"POST ", b"/index.html", b" HTTP/1.1\r\n", b"Host: www.example.com\r\n",
               b"User-Agent: Mozilla/5.0 (X11; Linux x86_64)\r\n", b"Accept: */*\r\n", b"Connection: keep-alive\r\n",
               b"Cookie: session=", b"&", b"=", b"id", b"page", b"user", b"the ", b"and ", b"of ", b"to ", b"data",
               b"/images/", b".png", b".js", b"Content-Type: text/html\r\n", b"\r\n", b"q=search+terms",
               b"lang=en", b"static", b"api/v1/", b"json", b"200 OK", b"<html>", b"<div class=\"", b"\">",
               b"</div>", b"var x = ", b"function", b"(", b")", b";", b"0123", b"4567", b"89"]


def _fill_records(rng, length, kinds, probs, sources, rec_max=1460):
    """Stream of records of length U(0, rec_max); each record draws its bytes
    from sources[kind] at a random offset."""
    out = np.empty(length, dtype=np.uint8)
    pos = 0
    chunk = 1 << 22
    while pos < length:
        nrec = chunk // (rec_max // 2) + 2
        lens = rng.integers(0, rec_max + 1, size=nrec)
        kind = rng.choice(kinds, size=nrec, p=probs)
        ends = np.cumsum(lens)
        take = int(min(length - pos, ends[-1]))
        nrec_used = int(np.searchsorted(ends, take, side="left")) + 1
        lens, kind = lens[:nrec_used], kind[:nrec_used]
        starts = np.concatenate([[0], np.cumsum(lens)[:-1]])
        rec_id = np.repeat(np.arange(nrec_used), lens)[:take]
        local = np.arange(take) - starts[rec_id]
        seg = np.zeros(take, dtype=np.uint8)
        for k, src in enumerate(sources):
            m = kind[rec_id] == k
            if not m.any():
                continue
            offs = rng.integers(0, src.size, size=nrec_used)
            idx = (offs[rec_id[m]] + local[m]) % src.size
            seg[m] = src[idx]
        out[pos:pos + take] = seg
        pos += take
    return out


def _plant(rng, buf: np.ndarray, samplers, every: int):
    n = buf.size
    k = max(1, n // every)
    for _ in range(k):
        s = samplers[int(rng.integers(0, len(samplers)))](rng)
        if not s or len(s) >= n:
            continue
        at = int(rng.integers(0, n - len(s)))
        buf[at:at + len(s)] = np.frombuffer(s, dtype=np.uint8)


def snort_input(length: int = 256 << 20, seed: int = 2, patterns_seed: int = 2, n_patterns: int = 1000):
    """Packet payloads: records of 0-1460 B, 50% HTTP-like text, 30% uniform
    random bytes, 20% base64-ish; members of L(r) of 10% of the regexes
    planted about once per 64 KiB."""
    rng = np.random.default_rng(seed * 7919 + 1)
    pool = min(length, 8 << 20) + 1
    text = _text_pool(rng, pool, _HTTP_VOCAB)
    rnd = rng.integers(0, 256, size=pool, dtype=np.uint8)
    b64a = np.frombuffer(b"ABCDEFGHIJKLMNOPQRSTUVWXYZabcdefghijklmnopqrstuvwxyz0123456789+/", dtype=np.uint8)
    b64 = b64a[rng.integers(0, 64, size=pool)]
    buf = _fill_records(rng, length, [0, 1, 2], [0.5, 0.3, 0.2], [text, rnd, b64])
    _, samplers = snort_patterns(n_patterns, patterns_seed)
    chosen = [samplers[i] for i in rng.choice(len(samplers), size=max(1, len(samplers) // 10), replace=False)]
    _plant(rng, buf, chosen, 64 << 10)
    return buf


CONFIGS["snort"] = {
    "patterns": lambda n=1000, seed=2: snort_patterns(n, seed)[0],
    "input": lambda length=256 << 20, seed=2: snort_input(length, seed),
    "pattern_kw": ("n",),
    "input_kw": ("length",),
    "len": 256 << 20,
    "desc": "Snort-like: 1,000 regexes over 256 MiB synthetic packet payloads (seed 2)",
}


# ---------------------------------------------------------------------------
# config 3: ClamAV-like hex signatures + Brill-like word rules over text
# (Table 1: ClamAV length mean 359.7 / SD 310.7 chars; Brill 44.4 /
# 16.9)
# ---------------------------------------------------------------------------
def _syn_words(rng, n: int):
    """n synthetic lowercase words (2-10 letters), deterministic."""
    letters = b"etaoinshrdlcumwfgypbvkjxqz"
    freq = np.array([12.7, 9.1, 8.2, 7.5, 7.0, 6.7, 6.3, 6.1, 6.0, 4.3, 4.0, 2.8, 2.8, 2.4, 2.4, 2.2, 2.0, 2.0, 1.9,
                     1.5, 1.0, 0.8, 0.2, 0.2, 0.1, 0.1])
    freq = freq / freq.sum()
    out = set()
    while len(out) < n:
        k = int(rng.integers(2, 11))
        out.add(bytes(letters[int(i)] for i in rng.choice(26, size=k, p=freq)))
    return sorted(out)


def _zipf_text(rng, length: int, words, s: float = 1.1, line: int = 80) -> np.ndarray:
    ranks = np.arange(1, len(words) + 1, dtype=np.float64)
    p = ranks ** (-s)
    p /= p.sum()
    punct = [b" ", b" ", b" ", b" ", b" ", b", ", b". ", b"; "]
    out = bytearray()
    col = 0
    while len(out) < length:
        idx = rng.choice(len(words), size=4096, p=p)
        pk = rng.integers(0, len(punct), size=4096)
        for i, j in zip(idx, pk):
            w = words[int(i)] + punct[int(j)]
            out += w
            col += len(w)
            if col >= line:
                out += b"\n"
                col = 0
        if len(out) >= length:
            break
    return np.frombuffer(bytes(out[:length]), dtype=np.uint8).copy()


_TEXT_WORDS_SEED = 33


def text_words(n: int = 50000):
    """n synthetic words in Zipf-rank order (a seeded permutation)."""
    rng = np.random.default_rng(_TEXT_WORDS_SEED)
    w = _syn_words(rng, n)
    return [w[int(i)] for i in rng.permutation(len(w))]


def clamav_patterns(n: int = 1000, seed: int = 3):
    """Hex byte signatures, length lognormal mean 360 / SD 311 chars clipped to
    [16, 2048]; 10% with '.' or '.{0,32}' gaps."""
    rng = np.random.default_rng(seed)
    pats, samplers = [], []
    for _ in range(n):
        chars = _lognormal_len(rng, 360, 311, lo=16, hi=2048)
        nbytes = max(4, chars // 4)
        toks = []
        gap = rng.random() < 0.10
        left = nbytes
        while left > 0:
            seg = int(min(left, rng.integers(8, 40) if gap else left))
            b = bytes(rng.integers(0, 256, size=seg, dtype=np.uint8))
            toks.append(_Tok(b"".join(b"\\x%02x" % c for c in b), lambda g, b=b: b))
            left -= seg
            if gap and left > 0:
                if rng.random() < 0.5:
                    toks.append(_Tok(b".", lambda g: bytes([int(g.integers(0, 10))])))
                else:
                    k = int(rng.integers(1, 33))
                    toks.append(_quantified(b".", lambda g: b"a", 0, k, b"{0,%d}" % k))
        pats.append(b"".join(t.text for t in toks))
        samplers.append(lambda g, toks=toks: b"".join(t.sample(g) for t in toks))
    return pats, samplers


def brill_patterns(n: int = 1000, seed: int = 3):
    """Word-sequence rules (mean ~44 chars): alternations of words joined by
    '[ ]+' and optional '[a-z]+' wildcards."""
    rng = np.random.default_rng(seed * 101 + 7)
    words = text_words()
    top = words[:3000]
    pats, samplers = [], []
    for _ in range(n):
        target = _lognormal_len(rng, 44.4, 16.9, lo=10, hi=160)
        toks = []
        size = 0
        while size < target:
            if toks:
                toks.append(_Tok(b"[ ]+", lambda g: b" "))
            r = rng.random()
            if r < 0.5:
                w = top[int(rng.integers(0, len(top)))]
                t = _lit(w)
            elif r < 0.8:
                alts = [top[int(i)] for i in rng.integers(0, len(top), size=int(rng.integers(2, 5)))]
                t = _alt_tok(alts)
            else:
                t = _Tok(b"[a-z]+", lambda g: bytes(b"abcdefghijklmnopqrstuvwxyz"[int(i)]
                                                       for i in g.integers(0, 26, size=int(g.integers(1, 8)))))
            toks.append(t)
            size = sum(len(x.text) for x in toks)
        pats.append(b"".join(t.text for t in toks))
        samplers.append(lambda g, toks=toks: b"".join(t.sample(g) for t in toks))
    return pats, samplers


def clamav_brill_patterns(n_each: int = 1000, seed: int = 3):
    a, sa = clamav_patterns(n_each, seed)
    b, sb = brill_patterns(n_each, seed)
    return a + b, sa + sb


def text_input(length: int = 1 << 30, seed: int = 3, patterns_seed: int = 3, n_each: int = 1000,
               plant_every: int = 1 << 20):
    """Zipf(1.1) text over 50k synthetic words with punctuation and a newline
    every ~80 chars; members of the pattern set planted about once per MiB."""
    rng = np.random.default_rng(seed * 7919 + 3)
    pool = _zipf_text(rng, min(length, 8 << 20) + 1, text_words())
    reps = -(-length // pool.size)
    if reps > 1:
        offs = rng.integers(0, pool.size, size=reps)
        buf = np.concatenate([np.roll(pool, -int(o)) for o in offs])[:length].copy()
    else:
        buf = pool[:length].copy()
    _, samplers = clamav_brill_patterns(n_each, patterns_seed)
    _plant(rng, buf, samplers, plant_every)
    return buf


CONFIGS["clamav"] = {
    "patterns": lambda n=1000, seed=3: clamav_brill_patterns(n, seed)[0],
    "input": lambda length=1 << 30, seed=3: text_input(length, seed),
    "pattern_kw": ("n",),
    "input_kw": ("length",),
    "len": 1 << 30,
    "desc": "ClamAV/Brill-like: 1,000 hex signatures + 1,000 word rules over 1 GiB text (seed 3)",
}


# ---------------------------------------------------------------------------
# config 4: Dotstar-like + PROSITE/Protomata-like motifs (Table 1 Protomata
# length mean 96.5 / SD 36.2) over amino-acid text and long lines
# ---------------------------------------------------------------------------
_AMINO = b"ACDEFGHIKLMNPQRSTVWY"
_AMINO_FREQ = np.array([8.25, 1.37, 5.45, 6.75, 3.86, 7.07, 2.27, 5.96, 5.84, 9.66, 2.42, 4.06, 4.70, 3.93, 5.53,
                        6.56, 5.34, 6.87, 1.08, 2.92])
_AMINO_FREQ = _AMINO_FREQ / _AMINO_FREQ.sum()
_AMINO_CLASSES = [b"[ILMV]", b"[FYW]", b"[KR]", b"[DE]", b"[ST]", b"[AG]", b"[NQ]", b"[^P]", b"[^C]"]


def _amino_class_members(text: bytes) -> bytes:
    if text.startswith(b"[^"):
        return bytes(c for c in _AMINO if c != text[2])
    return text[1:-1]


def dotstar_patterns(n: int = 1000, seed: int = 4):
    """3-6 literal segments of 4-12 bytes joined by '.*' (p = 0.3), else by
    '[^\\n]*' or '.{0,k}'."""
    rng = np.random.default_rng(seed)
    pats, samplers = [], []
    alpha = b"abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789"
    for _ in range(n):
        toks = []
        for si in range(int(rng.integers(3, 7))):
            if si:
                r = rng.random()
                if r < 0.3:
                    toks.append(_quantified(b".", lambda g: b"x", 0, -1, b"*"))
                elif r < 0.65:
                    toks.append(_quantified(rb"[^\n]", lambda g: b"y", 0, -1, b"*"))
                else:
                    k = int(rng.integers(1, 64))
                    toks.append(_quantified(b".", lambda g: b"z", 0, k, b"{0,%d}" % k))
            w = bytes(alpha[int(i)] for i in rng.integers(0, len(alpha), size=int(rng.integers(4, 13))))
            toks.append(_lit(w))
        pats.append(b"".join(t.text for t in toks))
        samplers.append(lambda g, toks=toks: b"".join(t.sample(g) for t in toks))
    return pats, samplers


def protomata_patterns(n: int = 1000, seed: int = 4):
    """PROSITE-like motifs over the 20 amino acids: letters, classes such as
    [ILMV] and [^P], '.', '.{2,4}'; length mean 96.5 / SD 36.2 chars."""
    rng = np.random.default_rng(seed * 101 + 9)
    pats, samplers = [], []
    for _ in range(n):
        target = _lognormal_len(rng, 96.5, 36.2, lo=12, hi=300)
        toks = []
        size = 0
        while size < target:
            r = rng.random()
            if r < 0.45:
                c = bytes([_AMINO[int(rng.choice(20, p=_AMINO_FREQ))]])
                t = _lit(c)
            elif r < 0.8:
                cl = _AMINO_CLASSES[int(rng.integers(0, len(_AMINO_CLASSES)))]
                m = _amino_class_members(cl)
                t = _Tok(cl, lambda g, m=m: bytes([m[int(g.integers(0, len(m)))]]))
            elif r < 0.9:
                t = _Tok(b".", lambda g: bytes([_AMINO[int(g.integers(0, 20))]]))
            else:
                lo = int(rng.integers(1, 4))
                hi = lo + int(rng.integers(1, 4))
                t = _quantified(b".", lambda g: bytes([_AMINO[int(g.integers(0, 20))]]), lo, hi,
                                b"{%d,%d}" % (lo, hi))
            toks.append(t)
            size += len(t.text)
        pats.append(b"".join(t.text for t in toks))
        samplers.append(lambda g, toks=toks: b"".join(t.sample(g) for t in toks))
    return pats, samplers


def dotstar_protomata_patterns(n_each: int = 1000, seed: int = 4):
    a, sa = dotstar_patterns(n_each, seed)
    b, sb = protomata_patterns(n_each, seed)
    return a + b, sa + sb


def amino_lines(rng, length: int) -> np.ndarray:
    """Amino-acid text in lines of 60-80 letters (background frequencies)."""
    body = _AMINO_np = np.frombuffer(_AMINO, dtype=np.uint8)[rng.choice(20, size=length, p=_AMINO_FREQ)]
    out = body.copy()
    pos = int(rng.integers(60, 81))
    while pos < length:
        out[pos] = 10
        pos += int(rng.integers(61, 82))
    return out


def long_lines(rng, length: int, words) -> np.ndarray:
    """Text with very long lines (100 KiB - 4 MiB without a newline)."""
    pool = _zipf_text(rng, min(length, 8 << 20) + 1, words, line=1 << 40)
    reps = -(-length // pool.size)
    buf = np.concatenate([np.roll(pool, -int(o)) for o in rng.integers(0, pool.size, size=reps)])[:length].copy() \
        if reps > 1 else pool[:length].copy()
    buf[buf == 10] = 32
    pos = int(rng.integers(100 << 10, 4 << 20))
    while pos < length:
        buf[pos] = 10
        pos += int(rng.integers(100 << 10, 4 << 20))
    return buf


def dotstar_input(length: int = 1 << 30, seed: int = 4, patterns_seed: int = 4, n_each: int = 1000,
                  plant_every: int = 256 << 10):
    """Half amino-acid lines, half long-line text (alternating 4 MiB stripes);
    members of the pattern set planted about once per 256 KiB."""
    rng = np.random.default_rng(seed * 7919 + 4)
    stripe = 4 << 20
    pool_len = min(length, 8 << 20) + stripe
    am = amino_lines(rng, pool_len)
    ll = long_lines(rng, pool_len, text_words())
    buf = np.empty(length, dtype=np.uint8)
    pos = 0
    k = 0
    while pos < length:
        src = am if k % 2 == 0 else ll
        n = min(stripe, length - pos)
        o = int(rng.integers(0, src.size - n + 1))
        buf[pos:pos + n] = src[o:o + n]
        pos += n
        k += 1
    _, samplers = dotstar_protomata_patterns(n_each, patterns_seed)
    _plant(rng, buf, samplers, plant_every)
    return buf


CONFIGS["dotstar"] = {
    "patterns": lambda n=1000, seed=4: dotstar_protomata_patterns(n, seed)[0],
    "input": lambda length=1 << 30, seed=4: dotstar_input(length, seed),
    "pattern_kw": ("n",),
    "input_kw": ("length",),
    "len": 1 << 30,
    "desc": "Dotstar/Protomata-like: 1,000 + 1,000 regexes over 1 GiB amino/long-line text (seed 4)",
}


# ---------------------------------------------------------------------------
# config 5: 10k regexes (2,500 per family, seeds 51-54) over 8 GiB made of
# four 2 GiB family inputs (seed 5)
# ---------------------------------------------------------------------------
def multi_patterns(n_each: int = 2500):
    a = snort_patterns(n_each, 51)[0]
    b = clamav_patterns(n_each // 2, 52)[0] + brill_patterns(n_each - n_each // 2, 52)[0]
    c = dotstar_patterns(n_each, 53)[0]
    d = protomata_patterns(n_each, 54)[0]
    return a + b + c + d


def multi_input(length: int = 8 << 30, seed: int = 5, part: int = None):
    """The 8 GiB stream = snort-like | text | long-line/amino | amino, 2 GiB
    each; `part` selects one quarter (generated independently, so a rank can
    build only its own)."""
    q = length // 4
    gens = [lambda n: snort_input(n, seed=seed * 10 + 1, patterns_seed=51, n_patterns=2500),
            lambda n: text_input(n, seed=seed * 10 + 2, patterns_seed=52, n_each=1250),
            lambda n: dotstar_input(n, seed=seed * 10 + 3, patterns_seed=53, n_each=1250),
            lambda n: amino_lines(np.random.default_rng(seed * 10 + 4), n)]
    if part is not None:
        return gens[part](q if part < 3 else length - 3 * q)
    return np.concatenate([gens[i](q if i < 3 else length - 3 * q) for i in range(4)])


CONFIGS["multi"] = {
    "patterns": lambda n=2500: multi_patterns(n),
    "input": lambda length=8 << 30, seed=5: multi_input(length, seed),
    "pattern_kw": ("n",),
    "input_kw": ("length",),
    "len": 8 << 30,
    "desc": "10k regexes (2,500 per family) over 8 GiB (seed 5)",
}
