"""Thin ctypes binding of libbc.so (include/bc.h) -- argument marshalling only.

Every step of the method runs in the CUDA kernels behind the C ABI; this module
converts numpy arrays / torch tensors to pointers and return codes to
exceptions.  There is no CPU fallback: if libbc.so is missing or no GPU is
present the calls raise.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbc.so")

BC_OK, BC_EINVAL, BC_ENOMEM, BC_ECUDA, BC_EINTERNAL = 0, -1, -2, -3, -4
BC_STRATEGY_WE, BC_STRATEGY_EP, BC_STRATEGY_HYBRID, BC_STRATEGY_SAMPLING = 0, 1, 2, 3
STRATEGIES = {"we": 0, "ep": 1, "hybrid": 2, "sampling": 3}
BC_ENGINE_AUTO, BC_ENGINE_PER_SOURCE, BC_ENGINE_BATCHED, BC_ENGINE_GROUP = 0, 1, 2, 3
ENGINES = {"auto": 0, "per_source": 1, "batched": 2, "group": 3}
BATCH_WIDTH = 64  # sources per batch of the batched engine

EXPORTED = ("bc_graph_create", "bc_compute", "bc_compute_device", "bc_single_source",
            "bc_trace_source", "bc_batch_sources", "bc_default_options", "bc_set_options", "bc_get_options",
            "bc_get_stats", "bc_destroy", "bc_last_error")


class bc_options(ctypes.Structure):
    _fields_ = [("strategy", ctypes.c_int32), ("alpha", ctypes.c_int32), ("beta", ctypes.c_int32),
                ("gamma", ctypes.c_double), ("n_samps", ctypes.c_int32),
                ("ep_min_frontier", ctypes.c_int32), ("inflight", ctypes.c_int32),
                ("backward_we", ctypes.c_int32), ("block_threads", ctypes.c_int32),
                ("seq_max_deg", ctypes.c_int32), ("level_store", ctypes.c_int32),
                ("warp_max_deg", ctypes.c_int32), ("l2_persist", ctypes.c_int32),
                ("sort_frontier", ctypes.c_int32), ("extrapolate", ctypes.c_int32),
                ("normalize", ctypes.c_int32), ("succ_bits", ctypes.c_int32),
                ("engine", ctypes.c_int32), ("batch_levels", ctypes.c_int32),
                ("hub_chunk", ctypes.c_int32), ("group_ctas", ctypes.c_int32)]


class bc_stats(ctypes.Structure):
    _fields_ = [("sources", ctypes.c_int64), ("levels", ctypes.c_int64),
                ("we_levels", ctypes.c_int64), ("ep_levels", ctypes.c_int64),
                ("n_reached", ctypes.c_int64), ("arcs_reached", ctypes.c_int64),
                ("dag_arcs", ctypes.c_int64), ("arcs_scanned", ctypes.c_int64),
                ("sampling_ep", ctypes.c_int32), ("sampling_median", ctypes.c_int32),
                ("sigma_inexact", ctypes.c_int32), ("inflight", ctypes.c_int32),
                ("kernel_launches", ctypes.c_int32), ("bc_kernel_launches", ctypes.c_int32),
                ("kernel_ms", ctypes.c_double), ("phase_cycles", ctypes.c_int64 * 4),
                ("batches", ctypes.c_int64), ("batch_overflows", ctypes.c_int64),
                ("engines", ctypes.c_int32), ("pad_", ctypes.c_int32), ("dist_sum", ctypes.c_int64),
                ("handovers", ctypes.c_int64), ("group_wait_cycles", ctypes.c_int64),
                ("group_mode", ctypes.c_int32), ("pad2_", ctypes.c_int32)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_}
        d["phase_cycles"] = list(self.phase_cycles)
        return d


class BCError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libbc error {code}: {msg}")
        self.code = code


_lib = None
_vp = ctypes.c_void_p
_i32p = ctypes.POINTER(ctypes.c_int32)
_i64p = ctypes.POINTER(ctypes.c_int64)
_f64p = ctypes.POINTER(ctypes.c_double)
_u8p = ctypes.POINTER(ctypes.c_uint8)


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libbc.so; raises if it has not been built (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("BC_LIBBC", path)  # alternative build (tuning experiments)
    if not os.path.exists(path):
        raise RuntimeError(f"{path} not found: build it with `make` or __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    lib.bc_graph_create.argtypes = [ctypes.c_int32, ctypes.c_int64, _i64p, _i32p, ctypes.c_int,
                                    ctypes.c_int, ctypes.POINTER(_vp)]
    lib.bc_compute.argtypes = [_vp, _i32p, ctypes.c_int64, _f64p]
    lib.bc_compute_device.argtypes = [_vp, _vp, ctypes.c_int64, _vp, _vp]
    lib.bc_single_source.argtypes = [_vp, ctypes.c_int32, _i32p, _f64p, _f64p, _u8p,
                                     ctypes.c_int32, _i32p]
    lib.bc_trace_source.argtypes = [_vp, ctypes.c_int32, _i32p, _i64p, _i64p, ctypes.c_int32, _i32p]
    lib.bc_batch_sources.argtypes = [_vp, _i32p, ctypes.c_int32, _i32p, _f64p, _f64p]
    lib.bc_default_options.argtypes = [ctypes.POINTER(bc_options)]
    lib.bc_default_options.restype = None
    lib.bc_set_options.argtypes = [_vp, ctypes.POINTER(bc_options)]
    lib.bc_get_options.argtypes = [_vp, ctypes.POINTER(bc_options)]
    lib.bc_get_stats.argtypes = [_vp, ctypes.POINTER(bc_stats)]
    lib.bc_destroy.argtypes = [_vp]
    lib.bc_destroy.restype = None
    lib.bc_last_error.argtypes = []
    lib.bc_last_error.restype = ctypes.c_char_p
    for name in ("bc_graph_create", "bc_compute", "bc_compute_device", "bc_single_source",
                 "bc_trace_source", "bc_batch_sources", "bc_set_options", "bc_get_options",
                 "bc_get_stats"):
        getattr(lib, name).restype = ctypes.c_int
    _lib = lib
    return lib


def _check(rc: int):
    if rc != BC_OK:
        raise BCError(rc, bc_last_error())


def _ptr(a: Optional[np.ndarray], t):
    return None if a is None else a.ctypes.data_as(t)


# ----------------------------------------------------------- C-named wrappers


def bc_last_error() -> str:
    return load_library().bc_last_error().decode(errors="replace")


def bc_graph_create(n: int, row_offsets: np.ndarray, col_indices: np.ndarray,
                    directed: bool = False, device: int = 0) -> int:
    lib = load_library()
    ro = np.ascontiguousarray(row_offsets, dtype=np.int64)
    col = np.ascontiguousarray(col_indices, dtype=np.int32)
    if ro.size != n + 1:
        raise BCError(BC_EINVAL, "row_offsets must have n+1 entries")
    h = _vp()
    _check(lib.bc_graph_create(int(n), int(col.size), _ptr(ro, _i64p), _ptr(col, _i32p),
                               int(bool(directed)), int(device), ctypes.byref(h)))
    return h.value


def bc_compute(handle: int, sources: Optional[np.ndarray], bc_out: np.ndarray) -> np.ndarray:
    """Host in / host out; bc_out (float64[n]) is overwritten and returned."""
    lib = load_library()
    assert bc_out.dtype == np.float64 and bc_out.flags.c_contiguous
    if sources is None:
        _check(lib.bc_compute(_vp(handle), None, 0, _ptr(bc_out, _f64p)))
    else:
        src = np.ascontiguousarray(sources, dtype=np.int32)
        _check(lib.bc_compute(_vp(handle), _ptr(src, _i32p), int(src.size), _ptr(bc_out, _f64p)))
    return bc_out


def bc_compute_device(handle: int, d_sources_ptr: Optional[int], k: int, d_bc_ptr: int,
                      stream_ptr: Optional[int] = None):
    _check(load_library().bc_compute_device(_vp(handle), _vp(d_sources_ptr) if d_sources_ptr else None,
                                            int(k), _vp(d_bc_ptr), _vp(stream_ptr) if stream_ptr else None))


def bc_single_source(handle: int, n: int, s: int, max_levels: Optional[int] = None):
    lib = load_library()
    d = np.empty(n, dtype=np.int32)
    sigma = np.empty(n, dtype=np.float64)
    delta = np.empty(n, dtype=np.float64)
    ml = n + 1 if max_levels is None else max_levels
    modes = np.zeros(max(ml, 1), dtype=np.uint8)
    nl = ctypes.c_int32(0)
    _check(lib.bc_single_source(_vp(handle), int(s), _ptr(d, _i32p), _ptr(sigma, _f64p),
                                _ptr(delta, _f64p), _ptr(modes, _u8p), int(ml), ctypes.byref(nl)))
    L = nl.value
    return dict(d=d, sigma=sigma, delta=delta, level_modes=modes[:min(L, ml)].copy(), num_levels=L)


def bc_trace_source(handle: int, s: int, max_levels: int = 1 << 16) -> dict:
    """Per-level frontier sizes and forward/backward SM cycles of one source (N2)."""
    lib = load_library()
    ls = np.zeros(max_levels, dtype=np.int32)
    fc = np.zeros(max_levels, dtype=np.int64)
    bcyc = np.zeros(max_levels, dtype=np.int64)
    nl = ctypes.c_int32(0)
    _check(lib.bc_trace_source(_vp(handle), int(s), _ptr(ls, _i32p), _ptr(fc, _i64p),
                               _ptr(bcyc, _i64p), int(max_levels), ctypes.byref(nl)))
    L = min(nl.value, max_levels)
    return dict(level_sizes=ls[:L].copy(), fwd_cycles=fc[:L].copy(), bwd_cycles=bcyc[:L].copy(),
                num_levels=nl.value)


def bc_batch_sources(handle: int, n: int, sources) -> dict:
    """Per-source d / sigma / delta of one batch (1..64 sources) of the batched engine."""
    lib = load_library()
    src = np.ascontiguousarray(sources, dtype=np.int32)
    k = int(src.size)
    d = np.empty((k, n), dtype=np.int32)
    sigma = np.empty((k, n), dtype=np.float64)
    delta = np.empty((k, n), dtype=np.float64)
    _check(lib.bc_batch_sources(_vp(handle), _ptr(src, _i32p), k, _ptr(d, _i32p), _ptr(sigma, _f64p),
                                _ptr(delta, _f64p)))
    return dict(d=d, sigma=sigma, delta=delta)


def bc_default_options() -> bc_options:
    o = bc_options()
    load_library().bc_default_options(ctypes.byref(o))
    return o


def bc_set_options(handle: int, o: bc_options):
    _check(load_library().bc_set_options(_vp(handle), ctypes.byref(o)))


def bc_get_options(handle: int) -> bc_options:
    o = bc_options()
    _check(load_library().bc_get_options(_vp(handle), ctypes.byref(o)))
    return o


def bc_get_stats(handle: int) -> dict:
    st = bc_stats()
    _check(load_library().bc_get_stats(_vp(handle), ctypes.byref(st)))
    return st.as_dict()


def bc_destroy(handle: Optional[int]):
    if handle:
        load_library().bc_destroy(_vp(handle))


# ------------------------------------------------------------ convenience class


class BCGraph:
    """Owns a bc_graph handle for one graph on one device."""

    def __init__(self, n: int, row_offsets, col_indices, directed: bool = False, device: int = 0,
                 **options):
        self.n = int(n)
        self.directed = bool(directed)
        self.device = int(device)
        self.handle = bc_graph_create(n, row_offsets, col_indices, directed, device)
        if options:
            self.set_options(**options)

    @classmethod
    def from_graph(cls, g, device: int = 0, **options) -> "BCGraph":
        return cls(g.n, g.row_offsets, g.col_indices, g.directed, device, **options)

    def set_options(self, **kw):
        o = bc_get_options(self.handle)
        for k, v in kw.items():
            if k == "strategy" and isinstance(v, str):
                v = STRATEGIES[v]
            if k == "engine" and isinstance(v, str):
                v = ENGINES[v]
            if not hasattr(o, k):
                raise KeyError(k)
            setattr(o, k, v)
        bc_set_options(self.handle, o)

    def options(self) -> dict:
        o = bc_get_options(self.handle)
        return {k: getattr(o, k) for k, _ in o._fields_}

    def compute(self, sources: Optional[np.ndarray] = None) -> np.ndarray:
        out = np.empty(self.n, dtype=np.float64)
        return bc_compute(self.handle, sources, out)

    def compute_device(self, sources, out, stream=None):
        """sources: int32 CUDA tensor or None; out: float64 CUDA tensor [n]; async."""
        k = self.n if sources is None else int(sources.numel())
        sp = None if sources is None else sources.data_ptr()
        if sources is not None and k == 0:
            # an empty tensor has data_ptr() == 0, which the C ABI reads as "all n vertices";
            # k = 0 with any non-NULL pointer (never dereferenced) yields an all-zero BC
            sp = out.data_ptr()
        st = None if stream is None else stream.cuda_stream
        bc_compute_device(self.handle, sp, k, out.data_ptr(), st)
        return out

    def single_source(self, s: int, max_levels: Optional[int] = None) -> dict:
        return bc_single_source(self.handle, self.n, s, max_levels)

    def batch_sources(self, sources) -> dict:
        return bc_batch_sources(self.handle, self.n, sources)

    def trace_source(self, s: int, max_levels: int = 1 << 16) -> dict:
        return bc_trace_source(self.handle, s, max_levels)

    def stats(self) -> dict:
        return bc_get_stats(self.handle)

    def close(self):
        if getattr(self, "handle", None):
            bc_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
