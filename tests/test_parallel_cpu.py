"""Host-side multi-GPU protocol (paper_conf_micro_ge0025_b200/parallel.py) on
CPU with the gloo backend, world sizes 2 and 3.

The GPU matching is replaced by a small exact model of a chunk's boundary
state so that the protocol -- halo exchange by all_gather, speculative zero-state
match, state resolution by all_gather rounds, rematch only where the true
incoming state differs, all-reduce of per-regex counts -- is checked end to
end across processes.
The model: the "regex" counts positions where the running count of byte 'a'
since the last 'z' is odd; the boundary state is that parity (a carried
state in the sense of DESIGN.md "Forwarded state").
"""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_micro_ge0025_b200 import parallel


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def model_match(data: bytes, state_in: int, lo: int = 0, hi: int = None):
    """(count, state_out) of the toy program over data[lo:hi] (data may hold
    halo bytes around it): positions i where the parity of 'a's since the
    last 'z' is odd (carried state), plus positions with data[i-1:i+1] == b"bc"
    (one byte of lookback) and data[i:i+2] == b"ca" (one byte of lookahead)."""
    hi = len(data) if hi is None else hi
    par = state_in
    n = 0
    for i in range(lo, hi):
        b = data[i]
        if b == ord("z"):
            par = 0
        elif b == ord("a"):
            par ^= 1
        n += par
        n += i > 0 and data[i - 1:i + 1] == b"bc"
        n += data[i:i + 2] == b"ca"
    return n, par


class FakeProg:
    """Stands in for parallel.ChunkMatcher's Program (CPU tensors): computes
    from the halo'd buffer it is given, so the halo exchange is exercised."""

    def __init__(self):
        self.boundary_bytes = 4
        self.lookback = 1
        self.lookahead = 1
        self.calls = []

    def _run(self, buf, length, halo_left, state):
        data = bytes(buf.tolist())
        return model_match(data, state, halo_left, halo_left + length)

    def match_chunk(self, buf, length, halo_left, halo_right, global_offset, state_in=None, state_out=None,
                    out=None):
        s_in = 0 if state_in is None else int(state_in[0])
        n, s_out = self._run(buf, length, halo_left, s_in)
        out["counts"][0] = n
        state_out[0] = s_out
        self.calls.append(("match", s_in))

    def rematch_chunk(self, buf, length, halo_left, halo_right, global_offset, assumed, true, state_out, out):
        n_old, _ = self._run(buf, length, halo_left, int(assumed[0]))
        n_new, s_out = self._run(buf, length, halo_left, int(true[0]))
        out["counts"][0] += n_new - n_old
        state_out[0] = s_out
        self.calls.append(("rematch", int(true[0])))


def _worker(rank, world, port, data, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        prog = FakeProg()
        cm = parallel.ChunkMatcher(prog, torch.device("cpu"), dist=dist)
        a, b = parallel.chunk_bounds(len(data), world, rank)
        chunk = torch.tensor(list(data[a:b]), dtype=torch.uint8)
        out = {"counts": torch.zeros(1, dtype=torch.int64), "digests": None}
        reruns = cm.match_stream_chunk(chunk, rank, world, out, a)
        q.put((rank, int(out["counts"][0]), reruns, prog.calls, cm.last["gather_rounds"]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_chunked_protocol_equals_whole_stream(world):
    rng = torch.Generator().manual_seed(world)
    alphabet = b"aazbc"
    data = bytes(alphabet[i] for i in torch.randint(0, len(alphabet), (3000,), generator=rng).tolist())
    data = data[:1000] + b"a" + b"b" * 999 + data[2000:]  # a parity carried across a chunk boundary
    # "bc" / "ca" pairs straddling the cuts (halo bytes needed on both sides)
    cuts = [parallel.chunk_bounds(len(data), world, r)[0] for r in range(1, world)]
    for j, c in enumerate(cuts):
        pair = b"bc" if j % 2 == 0 else b"ca"
        data = data[:c - 1] + pair + data[c + 1:]
    whole, _ = model_match(data, 0)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, data, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    # every rank holds the all-reduced total == the whole-stream count
    assert all(r[1] == whole for r in res), (whole, res)
    # rank r re-ran iff its true incoming state was not the assumed zero
    for rank, _, reruns, calls, rounds in res:
        a, _ = parallel.chunk_bounds(len(data), world, rank)
        _, true_in = model_match(data[:a], 0)
        assert reruns == (1 if rank > 0 and true_in != 0 else 0)
        if reruns:
            assert calls[-1] == ("rematch", true_in)
        assert 1 <= rounds <= world


def test_shard_patterns_is_a_balanced_partition():
    costs = [float(c) for c in [5, 1, 9, 3, 3, 7, 2, 8, 1, 4]]
    for world in (1, 2, 3, 4):
        shards = [parallel.shard_patterns(len(costs), world, r, costs) for r in range(world)]
        flat = sorted(i for s in shards for i in s)
        assert flat == list(range(len(costs)))
        loads = [sum(costs[i] for i in s) for s in shards]
        assert max(loads) - min(loads) <= max(costs)


def test_chunk_bounds_cover_the_stream():
    for n in (0, 1, 7, 1000):
        for world in (1, 2, 3, 8):
            cuts = [parallel.chunk_bounds(n, world, r) for r in range(world)]
            assert cuts[0][0] == 0 and cuts[-1][1] == n
            assert all(cuts[i][1] == cuts[i + 1][0] for i in range(world - 1))


def _shard_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        pats = [b"ab", b"abc", b"b", b"zz", b"ca", b"a", b"bca", b"q"]
        text = b"abcabzzcabcaqab" * 7
        mine = parallel.shard_patterns(len(pats), world, rank, costs=[float(len(p)) for p in pats])
        # this rank's "program": overlapping occurrence counts of its own patterns
        local = torch.tensor([sum(text.startswith(pats[i], k) for k in range(len(text))) for i in mine],
                             dtype=torch.int64)
        full = torch.zeros(len(pats), dtype=torch.int64)
        parallel.combine_shard_counts(dist, full, torch.tensor(mine, dtype=torch.int64), local)
        q.put((rank, full.tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_regex_shards_combine_to_the_whole_set(world):
    # bench.py --split regex: disjoint shards, scattered and all-reduced
    pats = [b"ab", b"abc", b"b", b"zz", b"ca", b"a", b"bca", b"q"]
    text = b"abcabzzcabcaqab" * 7
    whole = [sum(text.startswith(p, k) for k in range(len(text))) for p in pats]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(r[1] == whole for r in res), (whole, res)
