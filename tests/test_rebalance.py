"""Shift Rebalancing (Sec. 5.2; rx_rebalance.cpp) --
SURVEY 8(a) row a9.

CPU: the pass rewrites the paper's own example into the paper's result.
Figure 8/9 take the chain ((B1 >> 1) & B2 >> 1) & B3 -- `/abb/`
with B1 = 'a', B2 = B3 = 'b' -- to B5 = B2 << 1; B6 = B1 & B5; B7 = B3 << 2;
B8 = B6 & B7; B4 = B8 >> 2 (every SHIFT on an input, one shift at the end).

GPU: with RX_F_REBALANCE the whole path stays bit-exact against the CPU
oracle (random grammar, long carry chains, bounded repeats, and prefixes of
workload configs 2-4 with their full pattern sets).
"""
import re

import numpy as np
import pytest

import gen
import oracle

rx = pytest.importorskip("paper_conf_micro_ge0025_b200")


def _ir(prog):
    """{node id: (op, args...)} of the single-regex IR in rx_program_info."""
    nodes = {}
    for line in prog.info.splitlines():
        m = re.match(r"(\s*)v(\d+) = (\w+)(.*?)\s+\[", line)
        if m:
            nodes[int(m.group(2))] = (m.group(3), m.group(4).split())
            if not m.group(1):
                nodes["last"] = int(m.group(2))
    return nodes


def _live(nodes, root):
    seen, todo = set(), [root]
    while todo:
        v = todo.pop()
        if v in seen:
            continue
        seen.add(v)
        todo += [int(a[1:]) for a in nodes[v][1] if a.startswith("v")]
    return seen


def _out(nodes):
    # the output is the last top-level node in emission order
    return nodes["last"]


def test_abb_rebalanced_to_the_papers_figure_9():
    flags = rx.RX_F_REBALANCE | rx.RX_F_NO_PREFILTER | rx.RX_F_NO_GUARDS
    nodes = _ir(rx.Program([b"abb"], flags=flags))
    out = _out(nodes)
    op, args = nodes[out]
    # B4 = B8 >> 2: one Advance by 2 at the end
    assert op == "adv" and args[-1] == "k=2", nodes[out]
    live = _live(nodes, out)
    ops = sorted(nodes[v][0] for v in live)
    # B8 = B6 & B7, B6 = B1 & B5, B5 = B2 << 1, B7 = B3 << 2: two ANDs, two
    # lookaheads (by 1 and 2), the two classes, no other Advance
    assert ops.count("and") == 2 and ops.count("adv") == 1 and ops.count("look") == 2, ops
    looks = sorted(nodes[v][1][-1] for v in live if nodes[v][0] == "look")
    assert looks == ["k=1", "k=2"]
    # every lookahead reads a character class directly (an input of the DFG)
    for v in live:
        if nodes[v][0] == "look":
            assert nodes[int(nodes[v][1][0][1:])][0] == "cc"


def test_rebalancing_never_deepens_the_chain():
    # depth of the live DFG (longest op path) with and without the pass
    def depth(nodes, v, memo):
        if v not in memo:
            args = [int(a[1:]) for a in nodes[v][1] if a.startswith("v")]
            memo[v] = 1 + max((depth(nodes, a, memo) for a in args), default=0)
        return memo[v]

    for pat in [b"abb", b"abcdefg", b"a[0-9]x[a-z]yz", b"(ab|cd)ef"]:
        base = rx.RX_F_NO_PREFILTER | rx.RX_F_NO_GUARDS
        n0 = _ir(rx.Program([pat], flags=base))
        n1 = _ir(rx.Program([pat], flags=base | rx.RX_F_REBALANCE))
        assert depth(n1, _out(n1), {}) <= depth(n0, _out(n0), {}), pat


torch = pytest.importorskip("torch")


def _gpu_parity(pats, data, **kw):
    prog = rx.Program(pats, flags=rx.RX_F_REBALANCE, **kw)
    d = torch.frombuffer(bytearray(data), dtype=torch.uint8).cuda() if len(data) else \
        torch.zeros(0, dtype=torch.uint8, device="cuda")
    out = prog.match(d, dense=True)
    torch.cuda.synchronize()
    o = oracle.run_set(pats, bytes(data), dense=True)
    counts = out["counts"].cpu().numpy().view(np.uint64)
    assert int(out["status"].cpu()[0]) == 0
    bad = np.nonzero(counts != o["counts"])[0]
    assert bad.size == 0, [(pats[i][:60], int(counts[i]), int(o["counts"][i])) for i in bad[:5]]
    assert np.array_equal(out["digests"].cpu().numpy().view(np.uint64), o["digests"])
    dense = out["dense"].cpu().numpy().view(np.uint32)[:, : (len(data) + 31) // 32]
    assert np.array_equal(dense, o["dense"])
    return o


@pytest.mark.gpu
def test_rebalanced_fuzz_and_chains_bit_exact():
    rng = np.random.default_rng(77)
    pats = []
    while len(pats) < 60:
        p = gen.fuzz_pattern(rng)
        if len(p) <= 24:
            pats.append(p)
    pats += [b"abb", b"a(bc)*d", b"x.*y", b"q[^\\n]*z", b"[0-9]{3,9}x", b"abcdefghij", b"a[bc]{2,40}d"]
    for n in [1, 100, 4097, 40000]:
        _gpu_parity(pats, gen.fuzz_text(rng, n))
    body = b"a" + b"bc" * 30000 + b"d" + b"x" + b"abc" * 20000 + b"y\nq" + b"0" * 70000 + b"zabbabb"
    _gpu_parity(pats, body)


@pytest.mark.gpu
@pytest.mark.parametrize("config", ["snort", "clamav", "dotstar"])
def test_rebalanced_config_prefixes_bit_exact(config):
    if config == "snort":
        pats, data = gen.snort_patterns(1000, 2)[0], gen.snort_input((2 << 20) + 777, seed=2)
    elif config == "clamav":
        pats, data = gen.clamav_brill_patterns(1000, 3)[0], gen.text_input((3 << 20) + 55, seed=3)
    else:
        pats, data = gen.dotstar_protomata_patterns(1000, 4)[0], gen.dotstar_input((5 << 20) + 9, seed=4)
    prog = rx.Program(pats, flags=rx.RX_F_REBALANCE)
    d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
    out = prog.match(d, digests=True)
    torch.cuda.synchronize()
    o = oracle.run_set(pats, bytes(data))
    counts = out["counts"].cpu().numpy().view(np.uint64)
    assert int(out["status"].cpu()[0]) == 0
    bad = np.nonzero(counts != o["counts"])[0]
    assert bad.size == 0, [(pats[i][:60], int(counts[i]), int(o["counts"][i])) for i in bad[:5]]
    assert np.array_equal(out["digests"].cpu().numpy().view(np.uint64), o["digests"])
