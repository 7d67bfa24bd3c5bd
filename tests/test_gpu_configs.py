"""GPU parity on the workload configs 2-5 of BASELINE.json.

Every config's full pattern set, over a seeded prefix of its own synthetic
input that the oracle finishes in seconds (several MiB: thousands of windows,
every group's segments, a ragged tail), through the C ABI, compared with the
CPU oracle bit-exactly: every count and both position digests per regex
(integer work: DESIGN.md "Parity").  The full-size inputs, in the launch
configuration bench.py times, are covered by tests/test_gpu_fullsize.py.
"""
import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
rx = pytest.importorskip("paper_conf_micro_ge0025_b200")

pytestmark = pytest.mark.gpu


def _run(prog, data: np.ndarray):
    d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
    out = prog.match(d, digests=True)
    torch.cuda.synchronize()
    return (out["counts"].cpu().numpy().view(np.uint64), out["digests"].cpu().numpy().view(np.uint64),
            int(out["status"].cpu()[0]))


def _parity(pats, data, min_total=1, **opts):
    prog = rx.Program(pats, **opts)
    counts, digests, status = _run(prog, data)
    o = oracle.run_set(pats, bytes(data))
    assert status == 0
    bad = np.nonzero(counts != o["counts"])[0]
    assert bad.size == 0, [(pats[i][:60], int(counts[i]), int(o["counts"][i])) for i in bad[:5]]
    bad = np.nonzero((digests != o["digests"]).any(axis=1))[0]
    assert bad.size == 0, [pats[i][:60] for i in bad[:5]]
    assert int(o["counts"].sum()) >= min_total
    return o


def test_config2_snort_like_prefix():
    pats = gen.snort_patterns(1000, 2)[0]
    _parity(pats, gen.snort_input((4 << 20) + 12345, seed=2))


def test_config2_snort_like_prefix_bench_opts():
    # the bench's compile options for this workload (bench.PROGRAM_OPTS: K = 4,
    # 168 registers -> 12-warp pass-1 CTAs)
    import bench
    pats = gen.snort_patterns(1000, 2)[0]
    _parity(pats, gen.snort_input((4 << 20) + 12345, seed=2), **bench.PROGRAM_OPTS["snort"])


def test_config3_clamav_brill_prefix():
    pats = gen.clamav_brill_patterns(1000, 3)[0]
    # planted about once per MiB: 6 MiB holds several signature/rule members
    _parity(pats, gen.text_input((6 << 20) + 4321, seed=3))


def test_config4_dotstar_protomata_prefix():
    pats = gen.dotstar_protomata_patterns(1000, 4)[0]
    # 4 MiB stripes alternate amino-acid lines and 100 KiB-4 MiB lines without
    # '\n': 9 MiB covers both and a stripe boundary (long .* carry chains)
    _parity(pats, gen.dotstar_input((9 << 20) + 99, seed=4))


def test_config5_multi_10k_prefix():
    pats = gen.multi_patterns(2500)
    assert len(pats) == 10000
    # one MiB of each family's input (the 8 GiB stream's four quarters)
    _parity(pats, gen.multi_input(4 << 20, seed=5))
