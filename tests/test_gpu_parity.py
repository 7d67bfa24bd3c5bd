"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Integer/bitwise work: every match-end bit, every count and both position
digests must be identical.  Sizes span several windows,
segments and a ragged tail; edge cases: empty input, 1 byte, lengths that are
not multiples of 32, chains longer than a window, all-zero / all-0xFF / all
'\\n' inputs, a misaligned input pointer.
"""
import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

pytestmark = pytest.mark.gpu


def gpu_run(prog, data: bytes, dense=True, offset=0):
    buf = torch.zeros(len(data) + offset + 64, dtype=torch.uint8, device="cuda")
    if data:
        buf[offset:offset + len(data)] = torch.frombuffer(bytearray(data), dtype=torch.uint8).cuda()
    view = buf[offset:offset + len(data)]
    out = prog.match(view, dense=dense)
    torch.cuda.synchronize()
    res = {"counts": out["counts"].cpu().numpy().view(np.uint64),
           "digests": out["digests"].cpu().numpy().view(np.uint64),
           "status": int(out["status"].cpu()[0])}
    if dense:
        res["dense"] = out["dense"].cpu().numpy().view(np.uint32)[:, : (len(data) + 31) // 32]
    return res


def assert_parity(patterns, data, prog=None, dense=True, offset=0):
    prog = prog or rx.Program(patterns)
    g = gpu_run(prog, data, dense=dense, offset=offset)
    o = oracle.run_set(patterns, data, dense=dense)
    assert g["status"] == 0
    bad = np.nonzero(g["counts"] != o["counts"])[0]
    assert bad.size == 0, [(patterns[i], int(g["counts"][i]), int(o["counts"][i])) for i in bad[:5]]
    assert np.array_equal(g["digests"], o["digests"])
    if dense:
        for i in range(len(patterns)):
            if not np.array_equal(g["dense"][i], o["dense"][i]):
                w = np.nonzero(g["dense"][i] != o["dense"][i])[0]
                raise AssertionError(f"pattern {patterns[i]!r}: first differing word {w[:5]}")
    return g


def test_tiny_config_dense_bit_exact():
    pats = gen.tiny_patterns()
    data = gen.tiny_input()
    g = assert_parity(pats, data)
    assert int(g["counts"].sum()) > 0


@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 1000, 1023, 1024, 1025, 4097, 65536 + 7])
def test_tiny_patterns_ragged_lengths(n):
    data = gen.tiny_input(length=max(n, 1), long_chain=0)[:n]
    assert_parity(gen.tiny_patterns(), data)


def test_long_chain_across_many_windows():
    pats = [b"a(bc)*d", b"a[bc]*d", b"x.*y", b"(ab|c)+d", b"q[^\\n]*z"]
    body = b"a" + b"bc" * 30000 + b"d" + b"x" + b"abc" * 20000 + b"y\nq" + b"0" * 70000 + b"z"
    assert_parity(pats, body)


def test_fuzz_random_grammar():
    rng = np.random.default_rng(2024)
    pats = []
    while len(pats) < 60:
        p = gen.fuzz_pattern(rng)
        if len(p) <= 24:
            pats.append(p)
    prog = rx.Program(pats)
    for n in [5, 100, 3000, 40000]:
        t = gen.fuzz_text(rng, n)
        assert_parity(pats, t, prog=prog)


def test_byte_alphabet_edge_inputs():
    pats = [rb".", rb"[^a]", rb"\x00+", rb"[\x80-\xff]{2}", rb"\d\s", rb"\w+", rb"\W", rb"[^\n]*\n", rb"\xff.",
            rb"(\x00|\n)(\x00|\n)", rb"\x00\x00\x00", rb"[\x00-\xff]", rb"[^\x00]*"]
    prog = rx.Program(pats)
    rng = np.random.default_rng(8)
    for data in [b"\x00" * 5000, b"\xff" * 4099, b"\n" * 3000,
                 rng.integers(0, 256, size=50000, dtype=np.uint8).tobytes()]:
        assert_parity(pats, data, prog=prog)


def test_misaligned_input_pointer():
    data = gen.tiny_input(length=20000, long_chain=0)
    for off in (1, 3, 8):
        assert_parity(gen.tiny_patterns(), data, offset=off)


def _chunk_views(data: bytes, k: int, halo: int):
    n = len(data)
    cuts = [n * i // k for i in range(k + 1)]
    dev = torch.frombuffer(bytearray(data), dtype=torch.uint8).cuda()
    for i in range(k):
        a, b = cuts[i], cuts[i + 1]
        hl, hr = min(halo, a), min(halo, n - b)
        yield i, a, b, hl, hr, dev[a - hl:b + hr]


@pytest.mark.parametrize("k", [2, 5])
def test_chunked_equals_whole_sequential_state(k):
    pats = [b"a(bc)*d", b"a[bc]*d", b"x.*y", b"(ab|c)+d", b"q[^\\n]*z", b"abc", b"[0-9]+x"]
    data = (b"a" + b"bc" * 3000 + b"d" + b"x" + b"abc" * 2000 + b"y\nq" + b"0" * 7000 + b"z") * 3
    prog = rx.Program(pats)
    whole = gpu_run(prog, data, dense=False)
    halo = max(prog.lookback, prog.lookahead, 64)
    out = prog.alloc_outputs(0, dense=False)
    st = prog.new_state()
    for i, a, b, hl, hr, view in _chunk_views(data, k, halo):
        st_next = prog.new_state()
        prog.match_chunk(view, b - a, hl, hr, a, state_in=st if i else None, state_out=st_next, out=out,
                         accumulate=i > 0)
        st = st_next
    torch.cuda.synchronize()
    assert np.array_equal(out["counts"].cpu().numpy().view(np.uint64), whole["counts"])
    assert np.array_equal(out["digests"].cpu().numpy().view(np.uint64), whole["digests"])


def test_chunked_speculative_then_rematch():
    # all chunks in parallel with zero state, then the carry fix-up chain
    pats = [b"a(bc)*d", b"x.*y", b"q[^\\n]*z", b"(ab|c)+d"]
    data = (b"a" + b"bc" * 3000 + b"d" + b"x" + b"abc" * 2000 + b"y\nq" + b"0" * 7000 + b"z") * 2
    prog = rx.Program(pats)
    whole = gpu_run(prog, data, dense=False)
    halo = max(prog.lookback, prog.lookahead, 64)
    k = 4
    chunks = list(_chunk_views(data, k, halo))
    outs, outs_state = [], []
    for i, a, b, hl, hr, view in chunks:
        o = prog.alloc_outputs(0, dense=False)
        so = prog.new_state()
        prog.match_chunk(view, b - a, hl, hr, a, state_in=None if i == 0 else prog.new_state(), state_out=so, out=o)
        outs.append(o)
        outs_state.append(so)
    true_in = None
    for i, a, b, hl, hr, view in chunks:
        if i > 0:
            assumed = prog.new_state()
            if not torch.equal(true_in, assumed):
                prog.rematch_chunk(view, b - a, hl, hr, a, assumed, true_in, outs_state[i], outs[i])
        true_in = outs_state[i]
    torch.cuda.synchronize()
    tot = sum(o["counts"].cpu().numpy().view(np.uint64) for o in outs)
    dig = sum(o["digests"].cpu().numpy().view(np.uint64) for o in outs)
    assert np.array_equal(tot, whole["counts"])
    assert np.array_equal(dig, whole["digests"])


def test_match_list_equals_oracle_positions():
    # several segments per group (so the carry fix-up runs and lists only
    # the matches the speculative pass lacked), the 20 KB a(bc)*d chain
    # crossing segment boundaries, .* state crossing many windows
    pats = gen.tiny_patterns() + [rb"abcd.*xyz", rb"q[^z]*z", rb"(ab|cd)+e"]
    data = gen.tiny_input() * 8
    prog = rx.Program(pats)
    d = torch.frombuffer(bytearray(data), dtype=torch.uint8).cuda()
    out = prog.match(d, match_cap=1 << 20)
    torch.cuda.synchronize()
    assert int(out["status"].cpu()[0]) == 0
    reg, pos = prog.match_list(out)
    counts = out["counts"].cpu().numpy().view(np.uint64)
    assert reg.size == int(counts.sum()) > 0
    for r, p in enumerate(pats):
        want = oracle.Regex(p).run(data, dense=False, positions=True)["positions"]
        assert np.array_equal(pos[reg == r], want), p
    # truncated list: the total is still exact, the call reports it
    out2 = prog.match(d, match_cap=10)
    torch.cuda.synchronize()
    assert int(out2["match_total"].cpu()[0]) == reg.size
    with pytest.raises(rx.RxError):
        prog.match_list(out2)


def test_bounded_class_repeats_and_literal_runs():
    # C{n,m} lowered by doubling (O(log m) steps) and literal runs confirmed
    # byte by byte (Op::Lit) must give the chain's stream exactly: repeats
    # of every shape, runs crossing lanes / windows, literals at frame edges
    pats = [rb"ab[0-9]{0,7}x", rb"[a-c]{3,9}", rb"q[^\n]{5,40}z", rb"x[ab]{6,}y", rb"hello world literal run",
            rb"[a-z]{1,64}", rb"abcdefghij", rb"a{4,16}", rb"zz[0-9a-f]{2}(?:%[0-9a-f]{2}){0,5}q",
            rb"GET /index\.html HTTP/1\.[01]", rb"k[^\r\n]{0,64}\r\n", rb"[ab]{33,70}", rb"xyz.{0,100}uvw",
            rb"(?:foo|bar)baz[0-9]{2,12}done"]
    rng = np.random.default_rng(99)
    alpha = np.frombuffer(b"abcxyz0123456789qk \n\r%fhelowrdGETHTP/.", dtype=np.uint8)
    n = 300000
    buf = bytearray(alpha[rng.integers(0, alpha.size, size=n)].tobytes())
    plants = [b"hello world literal run", b"abcdefghij", b"GET /index.html HTTP/1.1", b"a" * 20, b"ab" * 40,
              b"q" + b"w" * 30 + b"z", b"k" + b"m" * 64 + b"\r\n", b"xyz" + b"-" * 90 + b"uvw",
              b"foobaz1234567done", b"zz0f%00%ab%ffq", b"x" + b"ab" * 10 + b"y"]
    for at in list(range(1000, n - 200, 1023)) + [n - 30]:
        s = plants[int(rng.integers(0, len(plants)))]
        at = min(at, n - len(s))
        buf[at:at + len(s)] = s
    assert_parity(pats, bytes(buf))


@pytest.mark.parametrize("max_regs", [96, 168, 184, 255])
def test_register_caps_and_cta_sizes(max_regs):
    # rx_options.max_regs picks the pass-1 CTA size (16 / 12 / 8 warps); every
    # cap must link (ptxas budgets warps in groups of four) and stay exact
    pats = gen.tiny_patterns() + [b"x.*y", b"q[^\\n]*z", b"abcdefgh"]
    data = gen.tiny_input(length=50000, long_chain=2000)
    assert_parity(pats, data, prog=rx.Program(pats, max_regs=max_regs))
