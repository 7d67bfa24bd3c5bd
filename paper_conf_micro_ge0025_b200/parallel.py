"""Multi-GPU partitioning (one process per GPU, torch.distributed).

The paper is single-GPU (intra-CTA barriers only); the
north star adds the two partitions that are natural for this path
(DESIGN.md "Multi-GPU"):

* regex-set sharding: rank r compiles its share of the patterns and scans
  the whole input; per-regex counts are combined with one all_reduce (no
  other exchange: the path has none);
* input chunking: rank r commits its chunk of one long stream, reading a
  halo of rx_max_lookback / rx_max_lookahead bytes from its neighbours.  The
  unbounded part of a chunk's dependency on the past is the boundary state
  (MatchStar carries, forwarded loop words); every rank first matches its
  chunk speculatively with a zero incoming state, then the states are
  resolved rank by rank (a broadcast per boundary) and a rank whose true
  incoming state differs re-runs its first windows (rx_rematch_chunk) until
  the two runs agree.  Counts are all-reduced.

All collectives go through torch.distributed (NCCL on GPUs, gloo in the CPU
tests); the matching itself is the C ABI.  `match_fn`/`rematch_fn` are
injectable so the host-side protocol can be tested without a GPU.
"""
from __future__ import annotations

from typing import Callable


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


def chunk_bounds(total: int, world: int, rank: int):
    return total * rank // world, total * (rank + 1) // world


def resolve_boundary_states(dist, rank: int, world: int, state_out, zero_state,
                            rematch: Callable[[object, object], None]):
    """Sequential carry resolution over ranks.

    state_out: this rank's end state after the speculative match (assumed
    incoming state = zero_state, except rank 0 whose incoming state is exact).
    rematch(assumed, true): re-run this rank's chunk with the true incoming
    state; updates state_out in place.  Returns the number of reruns here.
    """
    reruns = 0
    buf = zero_state.clone()
    for r in range(1, world):
        if rank == r - 1:
            buf.copy_(state_out)
        dist.broadcast(buf, src=r - 1)
        if rank == r:
            if not bool((buf == zero_state).all()):
                rematch(zero_state, buf.clone())
                reruns += 1
    return reruns


class ChunkMatcher:
    """Input chunking across ranks for one compiled Program (GPU path)."""

    def __init__(self, prog, device, dist=None):
        import torch
        import torch.distributed as tdist
        self.prog = prog
        self.dev = device
        self.dist = dist or tdist
        self.zero = torch.zeros(max(prog.boundary_bytes // 4, 1), dtype=torch.int32, device=device)
        self.state_out = torch.zeros_like(self.zero)

    def match_chunk(self, buf, length, halo_left, halo_right, global_offset, rank, world, out):
        """buf = [left halo | chunk | right halo] on this rank's device."""
        p = self.prog
        st_in = None if rank == 0 else self.zero
        p.match_chunk(buf, length, halo_left, halo_right, global_offset, state_in=st_in,
                      state_out=self.state_out, out=out)

        def rematch(assumed, true):
            p.rematch_chunk(buf, length, halo_left, halo_right, global_offset, assumed, true, self.state_out, out)

        reruns = 0
        if world > 1:
            reruns = resolve_boundary_states(self.dist, rank, world, self.state_out, self.zero, rematch)
            self.dist.all_reduce(out["counts"])
            if out.get("digests") is not None:
                self.dist.all_reduce(out["digests"])
        return reruns

    def match_stream_chunk(self, buf, rank, world, out, halo_left=0, halo_right=0, global_offset=0):
        length = buf.numel() - halo_left - halo_right
        return self.match_chunk(buf, length, halo_left, halo_right, global_offset, rank, world, out)
