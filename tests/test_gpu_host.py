"""rx_match_host (include/rx.h): the whole stream from pinned host memory,
copied in pieces that overlap the matching of the previous piece; pieces are
matched in order with halos and the exact incoming state, so every output
equals one rx_match over the whole stream -- and the CPU oracle."""
import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

pytestmark = pytest.mark.gpu


def _host(data):
    return torch.from_numpy(np.ascontiguousarray(data)).pin_memory()


@pytest.mark.parametrize("piece", [1024, 4096 + 1024, 1 << 16, 0])
def test_match_host_equals_device_match_and_oracle(piece):
    pats = gen.tiny_patterns() + gen.dotstar_protomata_patterns(1000, 4)[0][::20]
    data = gen.dotstar_input((3 << 20) + 333, seed=9).copy()
    # a while-loop carry crossing many piece boundaries
    run = np.frombuffer(b"a" + b"bc" * 100000 + b"d", dtype=np.uint8)
    data[1 << 20:(1 << 20) + run.size] = run
    prog = rx.Program(pats)
    n = data.size
    cap = 1 << 20
    h = prog.match_host(_host(data), piece_bytes=piece, dense=True, match_cap=cap)
    d = prog.match(torch.from_numpy(data).cuda(), dense=True, match_cap=cap)
    torch.cuda.synchronize()
    for k in ("counts", "digests", "dense"):
        assert torch.equal(h[k], d[k]), k
    assert int(h["status"].cpu()[0]) == 0
    rh, ph = prog.match_list(h)
    rd, pd = prog.match_list(d)
    assert np.array_equal(rh, rd) and np.array_equal(ph, pd)
    o = oracle.run_set(pats, bytes(data))
    assert np.array_equal(h["counts"].cpu().numpy().view(np.uint64), o["counts"])
    assert np.array_equal(h["digests"].cpu().numpy().view(np.uint64), o["digests"])
    assert int(o["counts"].sum()) > 0 and n > 3 << 20


def test_match_host_small_and_empty():
    pats = gen.tiny_patterns()
    prog = rx.Program(pats)
    for n in (0, 1, 31, 1025):
        data = np.frombuffer(gen.tiny_input(length=max(n, 1), long_chain=0)[:n], dtype=np.uint8)
        h = prog.match_host(_host(data.copy()), piece_bytes=1024)
        torch.cuda.synchronize()
        o = oracle.run_set(pats, bytes(data))
        assert np.array_equal(h["counts"].cpu().numpy().view(np.uint64), o["counts"])
        assert np.array_equal(h["digests"].cpu().numpy().view(np.uint64), o["digests"])
