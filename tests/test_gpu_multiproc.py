"""The multi-GPU chunk protocol (paper_conf_micro_ge0025_b200/parallel.py,
DESIGN.md "Multi-GPU") with the REAL kernels: 2 and 3 processes on one GPU
(gloo; the halo bytes and boundary states move through the host), each rank
holding one chunk of a stream, running rx_match_chunk / rx_rematch_chunk
through the C ABI.  Every rank must end with the whole stream's exact
per-regex counts and position digests: equal to one rx_match over the whole
stream and to the CPU oracle.

The processes only exchange host tensors, so no kernel ever waits on another
process's kernel (B200_PROFILING.md: do not stand in for more GPUs with ranks
that wait on each other on one GPU).  The input has lines far longer than a
chunk, so `.*` / `[^\\n]*` carries cross the cuts and the rematch path runs.
"""
import os
import socket

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _workload():
    pats = gen.dotstar_protomata_patterns(1000, 4)[0][::8] + gen.tiny_patterns()  # 250 + 4 regexes
    data = gen.dotstar_input(3 << 20, seed=4).copy()
    # every chunk cut of 2 and 3 ranks lies inside a planted while-loop carry:
    # 'a(bc)*d' spans it
    run = np.frombuffer(b"a" + b"bc" * 40000 + b"d", dtype=np.uint8)
    for cut in (len(data) // 3, len(data) // 2, 2 * len(data) // 3):
        data[cut - 30000:cut - 30000 + run.size] = run
    return pats, np.ascontiguousarray(data)


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ.setdefault("RX_CACHE_DIR", os.path.join(ROOT, ".rxcache"))
    try:
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_micro_ge0025_b200 import parallel
        pats, data = _workload()
        dev = torch.device("cuda", 0)
        prog = rx.Program(pats)
        a, b = parallel.chunk_bounds(len(data), world, rank)
        chunk = torch.from_numpy(data[a:b].copy()).to(dev)
        out = prog.alloc_outputs(b - a, dev, dense=False, digests=True)
        cm = parallel.ChunkMatcher(prog, dev, dist=dist)
        cm.match_stream_chunk(chunk, rank, world, out, a)
        torch.cuda.synchronize()
        q.put((rank, out["counts"].cpu().numpy().view(np.uint64).copy(),
               out["digests"].cpu().numpy().view(np.uint64).copy(), int(out["status"].cpu()[0]), cm.last, None))
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, None, None, -1, None, repr(e)))


@pytest.fixture(scope="module")
def whole():
    pats, data = _workload()
    prog = rx.Program(pats)
    d = torch.from_numpy(data).cuda()
    out = prog.match(d, digests=True)
    torch.cuda.synchronize()
    got = (out["counts"].cpu().numpy().view(np.uint64), out["digests"].cpu().numpy().view(np.uint64))
    ref = oracle.run_set(pats, bytes(data))
    assert np.array_equal(got[0], ref["counts"]) and np.array_equal(got[1], ref["digests"])
    assert int(ref["counts"].sum()) > 0
    return got


@pytest.mark.parametrize("world", [2, 3])
def test_chunk_protocol_real_kernels_equals_whole_stream(world, whole):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted((q.get(timeout=900) for _ in procs), key=lambda r: r[0])
    for p in procs:
        p.join(timeout=120)
    for rank, counts, digests, status, last, err in res:
        assert err is None, (rank, err)
        assert status == 0
        bad = np.nonzero(counts != whole[0])[0]
        assert bad.size == 0, (rank, bad[:8], counts[bad[:8]], whole[0][bad[:8]])
        assert np.array_equal(digests, whole[1]), rank
    # every cut lies inside a long carry chain: every rank but 0 rematched
    assert all(r[4]["reruns"] > 0 for r in res[1:]), [r[4] for r in res]
