"""Multi-GPU partitioning (one process per GPU, torch.distributed).

The paper is single-GPU (intra-CTA barriers only); the
north star adds the two partitions that are natural for this path
(DESIGN.md "Multi-GPU"):

* regex-set sharding (`shard_patterns`): rank r compiles its share of the
  patterns and scans the whole input; the per-regex results are disjoint, so
  the only exchange is gathering them at the end;
* input chunking (`ChunkMatcher`): rank r commits chunk r of one long
  stream.  Its halo -- the last rx_max_lookback bytes of chunk r-1 and the
  first rx_max_lookahead bytes of chunk r+1 -- is exchanged with one
  all_gather of every rank's edge bytes.  The unbounded part of a chunk's
  dependency on the past is the boundary state (MatchStar carries, forwarded
  loop words): every rank first matches its chunk with a zero incoming state
  (rank 0: the exact stream-start state), then all ranks all_gather their end
  states; rank r takes rank r-1's end state as its true incoming state and,
  where it differs from the state its results assumed, re-runs its first
  windows (rx_rematch_chunk) until the two runs agree.  A rematch can change
  a rank's own end state only if the difference outlived its whole chunk, so
  the gather repeats until no end state changes (one extra gather in the
  usual case, at most world rounds).  Counts and digests are then
  all-reduced (digests are sums of per-position hashes of global positions).

All collectives go through torch.distributed (NCCL on GPUs; gloo moves the
small tensors through the host); the matching itself is the C ABI.  The
Program is injectable so the protocol is testable without a GPU
(tests/test_parallel_cpu.py) and, on one GPU with two processes, against the
real kernels (tests/test_gpu_multiproc.py).
"""
from __future__ import annotations


def shard_patterns(n: int, world: int, rank: int, costs=None):
    """Indices of the patterns rank `rank` owns: greedy balance by cost
    (pattern length by default), deterministic on every rank."""
    costs = costs or [1.0] * n
    order = sorted(range(n), key=lambda i: -costs[i])
    load = [0.0] * world
    owner = [0] * n
    for i in order:
        r = min(range(world), key=lambda k: (load[k], k))
        owner[i] = r
        load[r] += costs[i]
    return [i for i in range(n) if owner[i] == rank]


def combine_shard_counts(dist, full, idx, local):
    """Regex sharding: scatter this rank's per-regex results `local` into the
    zeroed full-length vector `full` at the global regex ids `idx`, then sum
    over ranks (the shards are disjoint, so the sum is the whole set's)."""
    full.zero_()
    full.index_copy_(0, idx, local)
    all_reduce_sum(dist, full)
    return full


def chunk_bounds(total: int, world: int, rank: int):
    return total * rank // world, total * (rank + 1) // world


def _host_staged(dist):
    """gloo collectives take CPU tensors: stage device tensors through the host."""
    try:
        return dist.get_backend() == "gloo"
    except Exception:  # noqa: BLE001
        return True


def all_gather_same(dist, t):
    """all_gather of an equally shaped tensor from every rank -> list."""
    import torch
    world = dist.get_world_size()
    if _host_staged(dist) and t.device.type != "cpu":
        src = t.cpu()
        parts = [torch.empty_like(src) for _ in range(world)]
        dist.all_gather(parts, src)
        return [p.to(t.device) for p in parts]
    parts = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(parts, t)
    return parts


def all_reduce_sum(dist, t):
    if _host_staged(dist) and t.device.type != "cpu":
        src = t.cpu()
        dist.all_reduce(src)
        t.copy_(src)
    else:
        dist.all_reduce(t)


def exchange_halos(dist, chunk, halo_left: int, halo_right: int, rank: int, world: int, buf=None):
    """[left halo | chunk | right halo] for this rank: one all_gather of every
    rank's edge bytes (first `halo_right` and last `halo_left` bytes of its
    chunk; every chunk must be at least that long).  Rank 0 has no left halo
    (the stream starts there), rank world-1 no right halo.  Returns (buf,
    hl, hr) with the halo sizes actually used."""
    import torch
    n = chunk.numel()
    assert n >= max(halo_left, halo_right), "chunk shorter than the halo"
    hl = halo_left if rank > 0 else 0
    hr = halo_right if rank < world - 1 else 0
    if buf is None or buf.numel() != hl + n + hr:
        buf = torch.empty(hl + n + hr, dtype=torch.uint8, device=chunk.device)
    buf[hl:hl + n].copy_(chunk)
    if world > 1 and (halo_left or halo_right):
        edge = torch.cat([chunk[:halo_right], chunk[n - halo_left:]]) if halo_left else chunk[:halo_right].clone()
        parts = all_gather_same(dist, edge)
        if hl:
            buf[:hl].copy_(parts[rank - 1][halo_right:])
        if hr:
            buf[hl + n:].copy_(parts[rank + 1][:halo_right])
    return buf, hl, hr


def resolve_boundary_states(dist, rank: int, world: int, state_out, zero_state, rematch):
    """Carry resolution across ranks by all_gather (module docstring).

    state_out: this rank's end state after the speculative match (assumed
    incoming state = zero_state, except rank 0 whose incoming state is exact);
    rematch(assumed, true) re-runs this rank's chunk with the true incoming
    state and updates state_out in place.  Returns (reruns, gather rounds)."""
    import torch
    assumed = zero_state.clone()
    prev = None
    reruns = rounds = 0
    while True:
        states = all_gather_same(dist, state_out)
        rounds += 1
        if prev is not None and all(torch.equal(a, b) for a, b in zip(states, prev)):
            break
        if rank > 0 and not torch.equal(states[rank - 1], assumed):
            true = states[rank - 1].clone()
            rematch(assumed, true)
            assumed = true
            reruns += 1
        prev = states
        if rounds > world:  # cannot happen: each round fixes at least one more rank
            raise RuntimeError("boundary-state resolution did not converge")
    return reruns, rounds


class ChunkMatcher:
    """Input chunking across ranks for one compiled Program."""

    def __init__(self, prog, device, dist=None):
        import torch
        import torch.distributed as tdist
        self.prog = prog
        self.dev = device
        self.dist = dist or tdist
        self.zero = torch.zeros(max(prog.boundary_bytes // 4, 1), dtype=torch.int32, device=device)
        self.state_out = torch.zeros_like(self.zero)
        self.buf = None
        self.last = {}

    def match_chunk(self, buf, length, halo_left, halo_right, global_offset, rank, world, out):
        """buf = [left halo | chunk | right halo] on this rank's device;
        `out` ends up holding the whole stream's counts / digests on every
        rank.  Returns the number of rematches this rank ran."""
        p = self.prog
        st_in = None if rank == 0 else self.zero
        p.match_chunk(buf, length, halo_left, halo_right, global_offset, state_in=st_in,
                      state_out=self.state_out, out=out)

        def rematch(assumed, true):
            p.rematch_chunk(buf, length, halo_left, halo_right, global_offset, assumed, true, self.state_out, out)

        reruns, rounds = 0, 0
        if world > 1:
            reruns, rounds = resolve_boundary_states(self.dist, rank, world, self.state_out, self.zero, rematch)
            all_reduce_sum(self.dist, out["counts"])
            if out.get("digests") is not None:
                all_reduce_sum(self.dist, out["digests"])
        self.last = {"reruns": reruns, "gather_rounds": rounds}
        return reruns

    def match_stream_chunk(self, chunk, rank, world, out, global_offset):
        """One step of chunked matching: halo exchange, speculative match,
        boundary-state resolution, all-reduce.  `chunk` is this rank's chunk
        of the stream (device uint8), starting at `global_offset`."""
        p = self.prog
        self.buf, hl, hr = exchange_halos(self.dist, chunk, p.lookback, p.lookahead, rank, world, self.buf)
        return self.match_chunk(self.buf, chunk.numel(), hl, hr, global_offset, rank, world, out)
