"""ORACLE -- TEST INFRASTRUCTURE ONLY.

ctypes wrapper around oracle/liboracle.so (oracle/brandes_oracle.c): a plain
serial Brandes betweenness centrality on the CPU, written from PAPER.md (see the
C file's header for the passage-by-passage mapping).  Only tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this package.  It shares no code with the CUDA path and never imports it.

Parity status per function (DESIGN.md §3 lists the pins):
  bc / bc_push           pinned: Eq. (1) brute force (exact rationals), closed forms,
                         the sum-of-distances invariant, networkx.
  single_source d        pinned: scipy.sparse.csgraph BFS distances, lattice Manhattan.
  single_source sigma    pinned: brute-force path enumeration, lattice binomials, trees.
  single_source delta    pinned through BC (Eq. 3) and brute force per source.
  level sizes, counters  pinned: level sizes vs scipy distances; counters vs numpy.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "brandes_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_i32p = ctypes.POINTER(ctypes.c_int32)
_i64p = ctypes.POINTER(ctypes.c_int64)
_f64p = ctypes.POINTER(ctypes.c_double)


def build(force: bool = False) -> str:
    """Compile the oracle with gcc -O2 (plain C, no GPU)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-pthread",
                               "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        for name in ("oracle_bc", "oracle_bc_push"):
            f = getattr(lib, name)
            f.argtypes = [ctypes.c_int32, _i64p, _i32p, ctypes.c_int, _i32p, ctypes.c_int64,
                          _f64p, ctypes.c_int]
            f.restype = ctypes.c_int
        lib.oracle_single_source.argtypes = [ctypes.c_int32, _i64p, _i32p, ctypes.c_int,
                                             ctypes.c_int32, _i32p, _f64p, _f64p, _i32p,
                                             _i32p, _i64p]
        lib.oracle_single_source.restype = ctypes.c_int
        lib.oracle_single_source_push.argtypes = [ctypes.c_int32, _i64p, _i32p, ctypes.c_int,
                                                  ctypes.c_int32, _i32p, _f64p, _f64p]
        lib.oracle_single_source_push.restype = ctypes.c_int
        _lib = lib
    return _lib


def _p(a: Optional[np.ndarray], t):
    return None if a is None else a.ctypes.data_as(t)


def _csr(g):
    ro = np.ascontiguousarray(g.row_offsets, dtype=np.int64)
    col = np.ascontiguousarray(g.col_indices, dtype=np.int32)
    return ro, col


def bc(g, sources: Optional[np.ndarray] = None, nthreads: int = 1, variant: str = "pull") -> np.ndarray:
    """BC over `sources` (None = all vertices), halved if undirected."""
    lib = _load()
    ro, col = _csr(g)
    out = np.zeros(g.n, dtype=np.float64)
    src = None if sources is None else np.ascontiguousarray(sources, dtype=np.int32)
    k = 0 if src is None else src.size
    if src is not None and k == 0:
        return out  # an empty source list: the empty sum (never "all vertices")
    f = lib.oracle_bc if variant == "pull" else lib.oracle_bc_push
    rc = f(g.n, _p(ro, _i64p), _p(col, _i32p), int(g.directed), _p(src, _i32p), k,
           _p(out, _f64p), int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_bc failed rc={rc}")
    return out


def bc_push(g, sources=None, nthreads: int = 1) -> np.ndarray:
    return bc(g, sources, nthreads, variant="push")


def single_source(g, s: int):
    """Per-source export: dict(d, sigma, delta, level_sizes, num_levels, n_reached,
    arcs_reached, dag_arcs)."""
    lib = _load()
    ro, col = _csr(g)
    n = g.n
    d = np.empty(n, dtype=np.int32)
    sigma = np.empty(n, dtype=np.float64)
    delta = np.empty(n, dtype=np.float64)
    ls = np.zeros(n + 1, dtype=np.int32)
    nl = np.zeros(1, dtype=np.int32)
    cnt = np.zeros(3, dtype=np.int64)
    rc = lib.oracle_single_source(n, _p(ro, _i64p), _p(col, _i32p), int(g.directed), int(s),
                                  _p(d, _i32p), _p(sigma, _f64p), _p(delta, _f64p),
                                  _p(ls, _i32p), _p(nl, _i32p), _p(cnt, _i64p))
    if rc != 0:
        raise ValueError(f"oracle_single_source failed rc={rc}")
    L = int(nl[0])
    return dict(d=d, sigma=sigma, delta=delta, level_sizes=ls[:L].copy(), num_levels=L,
                n_reached=int(cnt[0]), arcs_reached=int(cnt[1]), dag_arcs=int(cnt[2]))


def single_source_push(g, s: int):
    lib = _load()
    ro, col = _csr(g)
    n = g.n
    d = np.empty(n, dtype=np.int32)
    sigma = np.empty(n, dtype=np.float64)
    delta = np.empty(n, dtype=np.float64)
    rc = lib.oracle_single_source_push(n, _p(ro, _i64p), _p(col, _i32p), int(g.directed), int(s),
                                       _p(d, _i32p), _p(sigma, _f64p), _p(delta, _f64p))
    if rc != 0:
        raise ValueError(f"oracle_single_source_push failed rc={rc}")
    return dict(d=d, sigma=sigma, delta=delta)
