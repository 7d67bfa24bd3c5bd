"""B200-native interleaved bitstream regex matching (BitGen's hot path).

Thin Python binding over the C ABI of ``include/rx.h`` (``librx.so``):
argument marshalling only.  Every step of matching runs in the generated
sm_100a kernels; there is no CPU fallback -- calls that compute raise
``RxError`` when the library or a CUDA device is missing.

PyTorch is used for device memory and streams only.
"""
from __future__ import annotations

import ctypes
import os
import threading

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "librx.so")
_lock = threading.Lock()
_lib = None

RX_OK, RX_EPARSE, RX_EUNSUPPORTED, RX_ETOOBIG, RX_EJIT, RX_ECUDA, RX_EINVAL, RX_ENOMEM, RX_EOVERFLOW = range(9)
RX_F_NO_REBALANCE, RX_F_NO_GUARDS, RX_F_NO_CACHE, RX_F_REBALANCE, RX_F_NO_PREFILTER = 1, 2, 4, 8, 16
RX_F_NO_MODEB, RX_F_STATS, RX_F_NO_LOCKSTEP, RX_F_MODEB, RX_F_LOCKSTEP_ROUND = 32, 64, 128, 256, 512

EXPORTED = ["rx_compile", "rx_free", "rx_num_regex", "rx_num_groups", "rx_max_lookback", "rx_max_lookahead",
            "rx_boundary_bytes", "rx_program_source", "rx_program_info", "rx_match", "rx_match_chunk",
            "rx_rematch_chunk", "rx_last_error", "rx_kernels_per_match", "rx_set_profiling", "rx_kernel_times", "rx_match_batch",
            "rx_prefilter_table", "rx_match_host"]


class RxError(RuntimeError):
    def __init__(self, status, msg, index=None, offset=None):
        super().__init__(f"rx status {status}: {msg}")
        self.status, self.index, self.offset = status, index, offset


class _Options(ctypes.Structure):
    _fields_ = [("interval", ctypes.c_uint32), ("max_regs", ctypes.c_uint32), ("group_size", ctypes.c_uint32),
                ("words_per_lane", ctypes.c_uint32), ("flags", ctypes.c_uint32), ("reserved", ctypes.c_uint32 * 3)]


class _Error(ctypes.Structure):
    _fields_ = [("pattern_index", ctypes.c_uint32), ("byte_offset", ctypes.c_uint32), ("msg", ctypes.c_char * 256)]


class _Output(ctypes.Structure):
    _fields_ = [("d_counts", ctypes.c_void_p), ("d_digests", ctypes.c_void_p), ("d_bitstreams", ctypes.c_void_p),
                ("pitch_words", ctypes.c_uint64), ("d_status", ctypes.c_void_p), ("d_matches", ctypes.c_void_p),
                ("match_cap", ctypes.c_uint64), ("d_match_total", ctypes.c_void_p)]


def lib_path() -> str:
    return _LIB_PATH


def load_library():
    """Load librx.so (building it in-tree first if it is missing)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(_LIB_PATH):
            from . import build as _b
            _b.build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp, u32, u64, sz = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_size_t
        lib.rx_compile.argtypes = [vp, vp, u32, ctypes.POINTER(_Options), ctypes.POINTER(vp), ctypes.POINTER(_Error)]
        lib.rx_compile.restype = ctypes.c_int
        lib.rx_free.argtypes = [vp]
        for f in ("rx_num_regex", "rx_num_groups", "rx_max_lookback", "rx_max_lookahead", "rx_kernels_per_match"):
            getattr(lib, f).argtypes = [vp]
            getattr(lib, f).restype = u32
        lib.rx_boundary_bytes.argtypes = [vp]
        lib.rx_boundary_bytes.restype = sz
        lib.rx_program_source.argtypes = [vp]
        lib.rx_program_source.restype = ctypes.c_char_p
        lib.rx_program_info.argtypes = [vp]
        lib.rx_program_info.restype = ctypes.c_char_p
        lib.rx_prefilter_table.argtypes = [vp, ctypes.POINTER(ctypes.POINTER(ctypes.c_uint32)),
                                           ctypes.POINTER(ctypes.c_uint32)]
        lib.rx_prefilter_table.restype = sz
        lib.rx_match.argtypes = [vp, vp, u64, vp, ctypes.POINTER(_Output)]
        lib.rx_match.restype = ctypes.c_int
        lib.rx_match_chunk.argtypes = [vp, vp, u64, u64, u64, u64, vp, vp, ctypes.c_int, vp, ctypes.POINTER(_Output)]
        lib.rx_match_chunk.restype = ctypes.c_int
        lib.rx_rematch_chunk.argtypes = [vp, vp, u64, u64, u64, u64, vp, vp, vp, vp, ctypes.POINTER(_Output)]
        lib.rx_rematch_chunk.restype = ctypes.c_int
        lib.rx_match_batch.argtypes = [vp, vp, vp, u32, vp, ctypes.POINTER(_Output)]
        lib.rx_match_batch.restype = ctypes.c_int
        lib.rx_match_host.argtypes = [vp, vp, u64, u64, vp, ctypes.POINTER(_Output)]
        lib.rx_match_host.restype = ctypes.c_int
        lib.rx_set_profiling.argtypes = [vp, ctypes.c_int]
        lib.rx_set_profiling.restype = ctypes.c_int
        lib.rx_kernel_times.argtypes = [vp, vp, vp, ctypes.c_int]
        lib.rx_kernel_times.restype = ctypes.c_int
        lib.rx_last_error.argtypes = []
        lib.rx_last_error.restype = ctypes.c_char_p
        _lib = lib
        return lib


def _check(status):
    if status != RX_OK:
        raise RxError(status, load_library().rx_last_error().decode("utf-8", "replace"))


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream_handle(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


class Program:
    """A compiled pattern set (rx_compile)."""

    def __init__(self, patterns, interval=None, max_regs=None, group_size=None, words_per_lane=None, flags=0):
        lib = load_library()
        pats = [p.encode("latin-1") if isinstance(p, str) else bytes(p) for p in patterns]
        self.patterns = pats
        n = len(pats)
        bufs = [ctypes.create_string_buffer(p, len(p) + 1) for p in pats]
        arr = (ctypes.c_void_p * max(n, 1))(*[ctypes.cast(b, ctypes.c_void_p) for b in bufs])
        lens = (ctypes.c_size_t * max(n, 1))(*[len(p) for p in pats])
        opt = _Options()
        opt.interval = 0 if interval is None else (0xFFFFFFFF if interval <= 0 else int(interval))
        opt.max_regs = int(max_regs or 0)
        opt.group_size = int(group_size or 0)
        opt.words_per_lane = int(words_per_lane or 0)
        opt.flags = int(flags)
        err = _Error()
        h = ctypes.c_void_p()
        st = lib.rx_compile(arr, lens, n, ctypes.byref(opt), ctypes.byref(h), ctypes.byref(err))
        if st != RX_OK:
            raise RxError(st, lib.rx_last_error().decode("utf-8", "replace"), err.pattern_index, err.byte_offset)
        self._h = h
        self._lib = lib

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            self._lib.rx_free(h)
            self._h = None

    # --- properties ---------------------------------------------------------
    @property
    def n_regex(self) -> int:
        return int(self._lib.rx_num_regex(self._h))

    @property
    def n_groups(self) -> int:
        return int(self._lib.rx_num_groups(self._h))

    @property
    def lookback(self) -> int:
        return int(self._lib.rx_max_lookback(self._h))

    @property
    def lookahead(self) -> int:
        return int(self._lib.rx_max_lookahead(self._h))

    @property
    def kernels_per_match(self) -> int:
        return int(self._lib.rx_kernels_per_match(self._h))

    @property
    def boundary_bytes(self) -> int:
        return int(self._lib.rx_boundary_bytes(self._h))

    @property
    def source(self) -> str:
        return self._lib.rx_program_source(self._h).decode()

    @property
    def info(self) -> str:
        return self._lib.rx_program_info(self._h).decode()

    # --- matching -----------------------------------------------------------
    def prefilter_table(self):
        """(blob u32 array copy, header dict) of the prefilter's device table, or None."""
        import numpy as np
        ptr = ctypes.POINTER(ctypes.c_uint32)()
        hdr = (ctypes.c_uint32 * 12)()
        n = self._lib.rx_prefilter_table(self._h, ctypes.byref(ptr), hdr)
        if not n:
            return None
        blob = np.ctypeslib.as_array(ptr, shape=(n,)).copy()
        keys = ["smem_words", "b4bits", "b3bits", "hbits", "o_b3", "o_b2", "o_ht", "o_ext", "o_fgoff", "o_fgent",
                "nfactor"]
        return blob, dict(zip(keys, list(hdr)[:11]))

    def alloc_outputs(self, length, device=None, dense=False, digests=True, match_cap=None):
        """Output buffers of rx_output.  match_cap: None = no match list;
        an int = a list of that many rx_match_t entries ({u32 regex, u32 pad,
        u64 pos}, held as int64[cap, 2]) plus its u64 total; 0 = total only."""
        import torch
        device = device or torch.device("cuda", torch.cuda.current_device())
        n = self.n_regex
        out = {"counts": torch.zeros(max(n, 1), dtype=torch.int64, device=device)[:n],
               "digests": torch.zeros((max(n, 1), 2), dtype=torch.int64, device=device)[:n] if digests else None,
               "status": torch.zeros(1, dtype=torch.int32, device=device)}
        if match_cap is not None:
            out["matches"] = torch.zeros((max(int(match_cap), 1), 2), dtype=torch.int64, device=device)
            out["match_cap"] = int(match_cap)
            out["match_total"] = torch.zeros(1, dtype=torch.int64, device=device)
        if dense:
            pitch = max((int(length) + 31) // 32, 1)
            out["dense"] = torch.zeros((max(n, 1), pitch), dtype=torch.int32, device=device)[:n]
            out["pitch"] = pitch
        else:
            out["dense"], out["pitch"] = None, 0
        return out

    def _out_struct(self, o):
        s = _Output()
        s.d_counts = o["counts"].data_ptr()
        s.d_digests = o["digests"].data_ptr() if o.get("digests") is not None else None
        s.d_bitstreams = o["dense"].data_ptr() if o.get("dense") is not None else None
        s.pitch_words = int(o.get("pitch") or 0)
        s.d_status = o["status"].data_ptr() if o.get("status") is not None else None
        if o.get("match_total") is not None:
            s.d_match_total = o["match_total"].data_ptr()
            s.d_matches = o["matches"].data_ptr() if o.get("match_cap") else None
            s.match_cap = int(o.get("match_cap") or 0)
        return s

    @staticmethod
    def match_list(out):
        """(regex ids u32[m], positions u64[m]) of the listed matches, sorted
        by (regex, position); raises if the list was truncated."""
        import numpy as np
        total = int(out["match_total"].cpu()[0])
        if total > out["match_cap"]:
            raise RxError(RX_EOVERFLOW, f"match list truncated: {total} matches > cap {out['match_cap']}")
        a = out["matches"][:total].cpu().numpy().view(np.uint64)
        reg, pos = (a[:, 0] & 0xFFFFFFFF).astype(np.uint32), a[:, 1].copy()
        order = np.lexsort((pos, reg))
        return reg[order], pos[order]

    def match(self, data, out=None, dense=False, digests=True, match_cap=None, stream=None):
        """Match a CUDA uint8 tensor; returns dict(counts=int64[n] (u64 bits),
        digests=int64[n,2], dense=int32[n, pitch] LSB-first, status, and with
        match_cap: matches / match_total -- see match_list())."""
        if out is None:
            out = self.alloc_outputs(data.numel(), data.device, dense=dense, digests=digests, match_cap=match_cap)
        s = self._out_struct(out)
        _check(self._lib.rx_match(self._h, _ptr(data), int(data.numel()), _stream_handle(stream), ctypes.byref(s)))
        return out

    def match_chunk(self, data, length, halo_left, halo_right, global_offset, state_in=None, state_out=None,
                    out=None, accumulate=False, dense=False, digests=True, match_cap=None, stream=None):
        """`data` is a CUDA uint8 tensor holding [halo_left | chunk(length) | halo_right]."""
        if out is None:
            out = self.alloc_outputs(length, data.device, dense=dense, digests=digests, match_cap=match_cap)
        s = self._out_struct(out)
        base = data.data_ptr() + int(halo_left)
        _check(self._lib.rx_match_chunk(self._h, ctypes.c_void_p(base), int(length), int(halo_left), int(halo_right),
                                        int(global_offset), _ptr(state_in), _ptr(state_out), int(bool(accumulate)),
                                        _stream_handle(stream), ctypes.byref(s)))
        return out

    def rematch_chunk(self, data, length, halo_left, halo_right, global_offset, state_assumed, state_true,
                      state_out, out, stream=None):
        s = self._out_struct(out)
        base = data.data_ptr() + int(halo_left)
        _check(self._lib.rx_rematch_chunk(self._h, ctypes.c_void_p(base), int(length), int(halo_left),
                                          int(halo_right), int(global_offset), _ptr(state_assumed),
                                          _ptr(state_true), _ptr(state_out), _stream_handle(stream),
                                          ctypes.byref(s)))
        return out

    def match_host(self, host, out=None, piece_bytes=0, dense=False, digests=True, match_cap=None, stream=None,
                   device=None):
        """rx_match_host: `host` a CPU uint8 tensor (pin_memory() for overlap);
        pipelined host-to-device copy + matching, result as match()."""
        import torch
        assert host.device.type == "cpu" and host.dtype == torch.uint8 and host.is_contiguous()
        device = device or torch.device("cuda", torch.cuda.current_device())
        if out is None:
            out = self.alloc_outputs(host.numel(), device, dense=dense, digests=digests, match_cap=match_cap)
        s = self._out_struct(out)
        _check(self._lib.rx_match_host(self._h, ctypes.c_void_p(host.data_ptr() if host.numel() else None),
                                       int(host.numel()), int(piece_bytes), _stream_handle(stream), ctypes.byref(s)))
        return out

    def match_batch(self, data, offsets, dense=False, digests=True, match_cap=None, stream=None, out=None):
        """rx_match_batch: `data` a CUDA uint8 tensor holding the streams back
        to back, `offsets` n_streams + 1 host ints.  Returns counts
        int64[n_streams, n_regex], digests int64[n_streams, n_regex, 2] (over
        positions relative to `data`),
        dense int32[n_streams, n_regex, pitch]; match-list positions are
        relative to `data`."""
        import numpy as np
        import torch
        offs = np.ascontiguousarray(np.asarray(offsets, dtype=np.uint64))
        ns = max(len(offs) - 1, 0)
        n, dev = self.n_regex, data.device
        max_len = int((offs[1:] - offs[:-1]).max()) if ns else 0
        if out is not None:  # reuse the buffers of an earlier call with the same shape
            s = self._out_struct(out)
            s.d_counts = out["counts_full"].data_ptr()
            _check(self._lib.rx_match_batch(self._h, _ptr(data), offs.ctypes.data_as(ctypes.c_void_p), ns,
                                            _stream_handle(stream), ctypes.byref(s)))
            return out
        counts_full = torch.zeros((max(ns, 1), max(n, 1)), dtype=torch.int64, device=dev)
        out = {"counts": counts_full[:ns, :n], "counts_full": counts_full,
               "digests": torch.zeros((max(ns, 1), max(n, 1), 2), dtype=torch.int64, device=dev)[:ns, :n]
               if digests else None,
               "status": torch.zeros(1, dtype=torch.int32, device=dev)}
        if match_cap is not None:
            out["matches"] = torch.zeros((max(int(match_cap), 1), 2), dtype=torch.int64, device=dev)
            out["match_cap"] = int(match_cap)
            out["match_total"] = torch.zeros(1, dtype=torch.int64, device=dev)
        if dense:
            pitch = max((max_len + 31) // 32, 1)
            out["dense"] = torch.zeros((max(ns, 1), max(n, 1), pitch), dtype=torch.int32, device=dev)[:ns, :n]
            out["pitch"] = pitch
        else:
            out["dense"], out["pitch"] = None, 0
        s = self._out_struct(out)
        s.d_counts = counts_full.data_ptr()  # an empty view may report a null pointer
        _check(self._lib.rx_match_batch(self._h, _ptr(data), offs.ctypes.data_as(ctypes.c_void_p), ns,
                                        _stream_handle(stream), ctypes.byref(s)))
        return out

    def set_profiling(self, on: bool = True):
        _check(self._lib.rx_set_profiling(self._h, int(bool(on))))

    def kernel_times(self, reset: bool = True):
        """{kernel: (total ms, launches)} for prefilter / pass1 / fixup (rx_kernel_times)."""
        ms = (ctypes.c_double * 3)()
        n = (ctypes.c_uint64 * 3)()
        _check(self._lib.rx_kernel_times(self._h, ms, n, int(bool(reset))))
        return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(("rx_prefilter", "rx_pass1", "rx_fixup"))}

    def new_state(self, device=None):
        import torch
        device = device or torch.device("cuda", torch.cuda.current_device())
        return torch.zeros(max(self.boundary_bytes // 4, 1), dtype=torch.int32, device=device)


def compile(patterns, **kw) -> Program:  # noqa: A001 (mirrors rx_compile)
    return Program(patterns, **kw)
