"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``)
and ``__graft_entry__.smoke()`` may import this package.  The product path in
``paper_conf_micro_ge0025_b200`` never imports it and shares no code with it.

The C source ``oracle/oracle.c`` is a Thompson-NFA simulator of the paper's
match-end bitstream definition (PAPER.md, all-match semantics) -- see
its header for the readings it follows.  This module is ctypes marshalling only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

RX_EPARSE, RX_EUNSUPPORTED, RX_ETOOBIG = 1, 2, 3


def build(force: bool = False) -> str:
    """Compile oracle.c into oracle/liboracle.so (plain gcc, -O2, pthreads)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-D_GNU_SOURCE", "-fPIC", "-shared", "-pthread",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB_PATH)
            u64, u32, sz = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_size_t
            vp = ctypes.c_void_p
            lib.orc_compile.argtypes = [ctypes.c_char_p, sz, ctypes.POINTER(vp), ctypes.POINTER(sz),
                                        ctypes.c_char_p, sz]
            lib.orc_compile.restype = ctypes.c_int
            lib.orc_free.argtypes = [vp]
            lib.orc_num_states.argtypes = [vp]
            lib.orc_nullable.argtypes = [vp]
            lib.orc_max_len.argtypes = [vp]
            lib.orc_max_len.restype = ctypes.c_int64
            lib.orc_run.argtypes = [vp, vp, u64, ctypes.c_int, ctypes.c_int, vp, vp, u64,
                                    ctypes.POINTER(u64), ctypes.POINTER(u64)]
            lib.orc_run.restype = u64
            lib.orc_run_set.argtypes = [vp, vp, u32, vp, u64, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                        vp, u64, vp, vp, ctypes.POINTER(u32)]
            lib.orc_run_set.restype = ctypes.c_int
            lib.orc_splitmix64.argtypes = [u64]
            lib.orc_splitmix64.restype = u64
            _lib = lib
    return _lib


def _as_bytes(p) -> bytes:
    return p.encode("latin-1") if isinstance(p, str) else bytes(p)


def _as_u8(data) -> np.ndarray:
    if isinstance(data, (bytes, bytearray, memoryview)):
        return np.frombuffer(bytes(data), dtype=np.uint8)
    a = np.ascontiguousarray(data, dtype=np.uint8)
    return a


class OracleError(ValueError):
    def __init__(self, code, index, offset, msg):
        super().__init__(f"pattern {index}: code {code} at byte {offset}: {msg}")
        self.code, self.index, self.offset = code, index, offset


class Regex:
    """One compiled oracle regex (Thompson NFA)."""

    def __init__(self, pattern):
        lib = _load()
        pat = _as_bytes(pattern)
        h = ctypes.c_void_p()
        at = ctypes.c_size_t(0)
        msg = ctypes.create_string_buffer(256)
        code = lib.orc_compile(pat, len(pat), ctypes.byref(h), ctypes.byref(at), msg, 256)
        if code:
            raise OracleError(code, 0, at.value, msg.value.decode("latin-1"))
        self._h = h
        self.pattern = pat

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.orc_free(h)
            self._h = None

    @property
    def num_states(self) -> int:
        return _load().orc_num_states(self._h)

    @property
    def nullable(self) -> bool:
        return bool(_load().orc_nullable(self._h))

    @property
    def max_len(self) -> int:
        """Longest string of L(r) (an upper bound on match length); -1 = unbounded."""
        return int(_load().orc_max_len(self._h))

    def run(self, data, use_cache: bool = True, max_states: int = 4096, dense: bool = True,
            positions: bool = False):
        """Returns dict(count, d1, d2, dense=u32[ceil(len/32)] LSB-first, positions=u64[])."""
        lib = _load()
        buf = _as_u8(data)
        n = int(buf.size)
        words = (n + 31) // 32
        dn = np.zeros(max(words, 1), dtype=np.uint32) if dense else None
        d1, d2 = ctypes.c_uint64(0), ctypes.c_uint64(0)
        cnt = lib.orc_run(self._h, buf.ctypes.data, n, int(use_cache), max_states,
                          dn.ctypes.data if dn is not None else None, None, 0,
                          ctypes.byref(d1), ctypes.byref(d2))
        out = {"count": int(cnt), "d1": int(d1.value), "d2": int(d2.value)}
        if dense:
            out["dense"] = dn[:words]
        if positions:
            pos = np.zeros(max(int(cnt), 1), dtype=np.uint64)
            lib.orc_run(self._h, buf.ctypes.data, n, int(use_cache), max_states, None, pos.ctypes.data,
                        int(cnt), None, None)
            out["positions"] = pos[: int(cnt)]
        return out


def check(pattern):
    """(code, offset, message) -- code 0 if the oracle's own parser accepts it."""
    lib = _load()
    pat = _as_bytes(pattern)
    h = ctypes.c_void_p()
    at = ctypes.c_size_t(0)
    msg = ctypes.create_string_buffer(256)
    code = lib.orc_compile(pat, len(pat), ctypes.byref(h), ctypes.byref(at), msg, 256)
    if code == 0:
        lib.orc_free(h)
    return code, at.value, msg.value.decode("latin-1")


def run_set(patterns, data, threads: int | None = None, use_cache: bool = True, max_states: int = 4096,
            dense: bool = False):
    """Whole pattern set over one input, a thread pool over regexes.

    Returns dict(counts=u64[n], digests=u64[n,2], dense=u32[n, ceil(len/32)] or None).
    """
    lib = _load()
    pats = [_as_bytes(p) for p in patterns]
    n = len(pats)
    buf = _as_u8(data)
    ln = int(buf.size)
    words = (ln + 31) // 32
    arr = (ctypes.c_char_p * max(n, 1))(*pats)
    lens = (ctypes.c_size_t * max(n, 1))(*[len(p) for p in pats])
    counts = np.zeros(max(n, 1), dtype=np.uint64)
    digests = np.zeros((max(n, 1), 2), dtype=np.uint64)
    dn = np.zeros((max(n, 1), max(words, 1)), dtype=np.uint32) if dense else None
    bad = ctypes.c_uint32(0)
    if threads is None:
        threads = os.cpu_count() or 1
    code = lib.orc_run_set(arr, lens, n, buf.ctypes.data, ln, int(threads), int(use_cache), max_states,
                           dn.ctypes.data if dn is not None else None, max(words, 1),
                           counts.ctypes.data, digests.ctypes.data, ctypes.byref(bad))
    if code:
        raise OracleError(code, bad.value, 0, "pattern rejected by the oracle parser")
    return {"counts": counts[:n], "digests": digests[:n],
            "dense": dn[:n, :words] if dense else None, "threads": int(threads)}


def positions_set(patterns, data, threads: int | None = None):
    """Sorted match-end positions (u64 arrays) of every pattern over one
    input, a thread pool over regexes (ctypes releases the GIL)."""
    from concurrent.futures import ThreadPoolExecutor
    buf = _as_u8(data)
    regs = [Regex(p) for p in patterns]
    with ThreadPoolExecutor(max_workers=threads or os.cpu_count() or 1) as ex:
        res = list(ex.map(lambda r: r.run(buf, dense=False, positions=True)["positions"], regs))
    return res


def splitmix64(x: int) -> int:
    return int(_load().orc_splitmix64(x))
