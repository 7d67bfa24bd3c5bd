"""CPU-side tests of the C ABI library (no GPU needed): it loads, exports
every symbol include/rx.h declares, compiles programs (parse -> IR -> NVRTC
sm_100a cubin) and reports errors consistently with the oracle's parser."""
import os
import re

import numpy as np
import pytest

import gen
import oracle
import paper_conf_micro_ge0025_b200 as rx

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "rx.h")).read()
    return sorted(set(re.findall(r"\b(rx_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    lib = rx.load_library()
    syms = declared_symbols()
    assert "rx_compile" in syms and "rx_match" in syms and "rx_match_chunk" in syms
    for s in syms:
        assert hasattr(lib, s), s
    assert set(syms) == set(rx.EXPORTED)


def test_compile_tiny_program_properties():
    p = rx.Program(gen.tiny_patterns())
    assert p.n_regex == 4 and p.n_groups >= 1
    assert p.boundary_bytes >= 4
    assert "extern \"C\" __global__" in p.source and "rx_pass1" in p.source
    assert p.kernels_per_match >= 1


def test_match_without_gpu_fails_loudly():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    p = rx.Program([b"abc"])
    with pytest.raises(Exception):
        p.match(torch.zeros(16, dtype=torch.uint8))


@pytest.mark.parametrize("pat", [b"^a", b"a$", b"a**", b"*a", b"(a", b"a)", b"[a", b"a{3,1}", b"\\1", b"a*?",
                                 b"(?=a)", b"\\bx", b"\\q", b"a{2000}"])
def test_rejects_like_the_oracle(pat):
    code, _, _ = oracle.check(pat)
    assert code != 0
    with pytest.raises(rx.RxError) as e:
        rx.Program([b"ok", pat])
    assert e.value.status == code, (pat, e.value.status, code)
    assert e.value.index == 1


def test_accepts_what_the_oracle_accepts():
    rng = np.random.default_rng(77)
    pats = [gen.fuzz_pattern(rng, depth=1) for _ in range(40)]
    pats += [rb"[]a]", rb"\.\*\x00", rb"[\x80-\xff]{2,5}", rb"a{,3}", rb"(?:ab|)c", rb"[^\n]*", rb"\W\S\D",
             rb"x{0}y", rb"(a|b|)*c"]
    for p in pats:
        assert oracle.check(p)[0] == 0, p
    rx.Program(pats)


def test_snort_like_patterns_all_compile_to_ir():
    pats = gen.snort_patterns(1000, 2)[0]
    for p in pats:
        assert oracle.check(p)[0] == 0
    # a slice through the full pipeline including NVRTC
    rx.Program(pats[:24])


def _struct_fields(src, name):
    body = re.search(r"struct " + name + r" \{(.*?)\n\};", src, re.S).group(1)
    body = re.sub(r"//[^\n]*", "", body)
    names = []
    for decl in body.split(";"):
        decl = decl.strip()
        if not decl:
            continue
        ty, rest = re.match(r"((?:const\s+)?(?:unsigned\s+)?(?:long\s+long|[A-Za-z0-9_]+)\s*\**)\s*(.*)", decl,
                            re.S).groups()
        for v in rest.split(","):
            names.append(v.strip().lstrip("*"))
    return names


def test_kernel_param_struct_mirrors_match():
    dev = open(os.path.join(ROOT, "paper_conf_micro_ge0025_b200", "csrc", "rx_device.cuh")).read()
    host = open(os.path.join(ROOT, "paper_conf_micro_ge0025_b200", "csrc", "rx_runtime.cpp")).read()
    a, b = _struct_fields(dev, "RxParams"), _struct_fields(host, "RxParamsHost")
    assert a == b, (a, b)


def test_match_batch_validates_offsets_before_any_launch():
    # host-side argument checks of rx_match_batch (include/rx.h) run before
    # any CUDA call, so the C entry point is testable without a GPU
    import ctypes
    import numpy as np
    p = rx.Program(gen.tiny_patterns())
    counts = np.zeros(3 * p.n_regex, dtype=np.uint64)
    o = rx._Output()
    o.d_counts = counts.ctypes.data
    bad = np.array([0, 40, 30, 64], dtype=np.uint64)
    st = p._lib.rx_match_batch(p._h, None, bad.ctypes.data_as(ctypes.c_void_p), 3, None, ctypes.byref(o))
    assert st == rx.RX_EINVAL and b"non-decreasing" in p._lib.rx_last_error()
    st = p._lib.rx_match_batch(p._h, None, None, 3, None, ctypes.byref(o))
    assert st == rx.RX_EINVAL


def test_match_host_validates_arguments_before_any_copy():
    # rx_match_host (include/rx.h) rejects null outputs / input and a short
    # dense pitch before touching the device, so it is checkable on CPU
    import ctypes
    import numpy as np
    p = rx.Program(gen.tiny_patterns())
    st = p._lib.rx_match_host(p._h, None, 16, 0, None, None)
    assert st == rx.RX_EINVAL
    counts = np.zeros(p.n_regex, dtype=np.uint64)
    o = rx._Output()
    o.d_counts = counts.ctypes.data
    st = p._lib.rx_match_host(p._h, None, 16, 0, None, ctypes.byref(o))
    assert st == rx.RX_EINVAL and b"null input" in p._lib.rx_last_error()
    buf = np.zeros(4096, dtype=np.uint8)
    dense = np.zeros(4, dtype=np.uint32)
    o.d_bitstreams = dense.ctypes.data
    o.pitch_words = 4
    st = p._lib.rx_match_host(p._h, buf.ctypes.data, buf.size, 0, None, ctypes.byref(o))
    assert st == rx.RX_EINVAL and b"pitch_words" in p._lib.rx_last_error()
