"""Seeded synthetic graph generators and the CSR builder.

This module is the ONE piece of code shared by the CUDA path's tests/bench and
the CPU oracle's tests: it produces inputs only and holds none of the method's
arithmetic (no BFS, no path counting, no dependency sums).

Graph classes follow the paper's benchmark families (Table II)
with the calibrations in SURVEY.md §4.6 / §8(d):

* R-MAT / Graph500 Kronecker  (kron_g500-logn20 [11]; A,B,C = .57,.19,.19)
* 2D 4-neighbour lattice and Delaunay triangulation (mesh class, delaunay_n20)
* random geometric graph, r = 0.55*sqrt(ln n / n)  (rgg_n_2_20 [21])
* Watts-Strogatz small world, k=10, p=0.2  (smallworld [37])

CSR convention: row_offsets int64[n+1], col_indices int32[nnz],
undirected graphs store both arcs of every edge, rows sorted ascending, no
self-loops, no duplicate arcs.  m (the TEPS edge count) is the number of
undirected edges = nnz/2.
"""
from __future__ import annotations

import ctypes
import dataclasses
import math
import os
import subprocess
from typing import Callable, Dict, Optional

import numpy as np


@dataclasses.dataclass
class Graph:
    name: str
    n: int
    row_offsets: np.ndarray  # int64[n+1]
    col_indices: np.ndarray  # int32[nnz]
    directed: bool = False

    @property
    def nnz(self) -> int:
        return int(self.row_offsets[-1])

    @property
    def m(self) -> int:
        """Edge count used by TEPS_BC = m*n/t: undirected edges."""
        return self.nnz if self.directed else self.nnz // 2

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_offsets)


# ------------------------------------------------------------------ native part

_HERE = os.path.dirname(os.path.abspath(__file__))
_NATIVE_SRC = os.path.join(_HERE, "graphgen_native.c")
_NATIVE_LIB = os.path.join(_HERE, "libgraphgen.so")
_native = None


def _threads() -> int:
    return max(1, min(32, len(os.sched_getaffinity(0))))


def native():
    """graphgen_native.c (gcc -O2, built on first use): counter-based R-MAT edge
    draw and a threaded CSR builder.  Input generation only."""
    global _native
    if _native is None:
        if (not os.path.exists(_NATIVE_LIB)
                or os.path.getmtime(_NATIVE_LIB) < os.path.getmtime(_NATIVE_SRC)):
            tmp = _NATIVE_LIB + f".{os.getpid()}.tmp"
            subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-pthread",
                                   "-o", tmp, _NATIVE_SRC])
            os.replace(tmp, _NATIVE_LIB)
        lib = ctypes.CDLL(_NATIVE_LIB)
        i64p = ctypes.POINTER(ctypes.c_int64)
        lib.gg_rmat_edges.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                      ctypes.c_double, ctypes.c_uint64, i64p, i64p, ctypes.c_int]
        lib.gg_rmat_edges.restype = None
        lib.gg_permutation.argtypes = [ctypes.c_int64, ctypes.c_uint64, i64p]
        lib.gg_permutation.restype = None
        lib.gg_csr_build.argtypes = [ctypes.c_int64, ctypes.c_int64, i64p, i64p, ctypes.c_int, i64p,
                                     ctypes.POINTER(ctypes.c_int32), ctypes.c_int]
        lib.gg_csr_build.restype = ctypes.c_int64
        _native = lib
    return _native


def _p64(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


# --------------------------------------------------------------------------- CSR


def csr_from_edges(n: int, u: np.ndarray, v: np.ndarray, directed: bool = False,
                   name: str = "graph") -> Graph:
    """Build a simple-graph CSR: drop self-loops, (symmetrise), dedupe, sort rows
    (threaded C builder; csr_from_edges_numpy is the reference it is tested against)."""
    u = np.ascontiguousarray(u, dtype=np.int64)
    v = np.ascontiguousarray(v, dtype=np.int64)
    cap = u.size if directed else 2 * u.size
    ro = np.zeros(n + 1, dtype=np.int64)
    col = np.empty(max(cap, 1), dtype=np.int32)
    nnz = native().gg_csr_build(int(n), int(u.size), _p64(u), _p64(v), int(directed), _p64(ro),
                                col.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), _threads())
    if nnz < 0:
        raise ValueError("edge endpoint out of range (or out of memory)")
    return Graph(name=name, n=n, row_offsets=ro, col_indices=col[:nnz].copy(), directed=directed)


def csr_from_edges_numpy(n: int, u: np.ndarray, v: np.ndarray, directed: bool = False,
                         name: str = "graph") -> Graph:
    """Reference numpy CSR builder (same contract as csr_from_edges)."""
    u = np.asarray(u, dtype=np.int64)
    v = np.asarray(v, dtype=np.int64)
    if u.size:
        if u.min() < 0 or v.min() < 0 or u.max() >= n or v.max() >= n:
            raise ValueError("edge endpoint out of range")
    keep = u != v
    u, v = u[keep], v[keep]
    if not directed:
        u, v = np.concatenate([u, v]), np.concatenate([v, u])
    key = np.unique(u * np.int64(n) + v)
    src = key // n
    dst = (key - src * n).astype(np.int32)
    counts = np.bincount(src, minlength=n).astype(np.int64)
    ro = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=ro[1:])
    return Graph(name=name, n=n, row_offsets=ro, col_indices=dst, directed=directed)


# --------------------------------------------------------------------- generators


def rmat_edges(scale: int, edgefactor: int = 16, a: float = 0.57, b: float = 0.19,
               c: float = 0.19, seed: int = 1, relabel: bool = True):
    """Raw R-MAT edge list (u, v) before the CSR builder; edge i is a pure function
    of (seed, i) (counter-based splitmix64 draw, graphgen_native.c)."""
    n = 1 << scale
    ne = edgefactor * n
    u = np.empty(ne, dtype=np.int64)
    v = np.empty(ne, dtype=np.int64)
    lib = native()
    lib.gg_rmat_edges(scale, ne, a, b, c, seed & 0xFFFFFFFFFFFFFFFF, _p64(u), _p64(v), _threads())
    if relabel:
        perm = np.empty(n, dtype=np.int64)
        lib.gg_permutation(n, seed & 0xFFFFFFFFFFFFFFFF, _p64(perm))
        u, v = perm[u], perm[v]
    return n, u, v


def rmat(scale: int, edgefactor: int = 16, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, seed: int = 1, relabel: bool = True,
         directed: bool = False, name: Optional[str] = None) -> Graph:
    """Graph500-style R-MAT/Kronecker generator (Chakrabarti et al. [11]).

    n = 2^scale vertices, edgefactor*n generated edges; per edge and per bit the
    quadrant is drawn with probabilities (a, b, c, 1-a-b-c); vertex labels are
    then randomly permuted.  Duplicates and self-loops are removed by the CSR
    builder (so m < edgefactor*n, and many vertices are isolated).
    """
    n, u, v = rmat_edges(scale, edgefactor, a, b, c, seed, relabel)
    return csr_from_edges(n, u, v, directed=directed,
                          name=name or f"rmat_s{scale}_ef{edgefactor}")


def lattice2d(rows: int, cols: int, name: Optional[str] = None) -> Graph:
    """4-neighbour grid; vertex (r, c) has id r*cols + c."""
    idx = np.arange(rows * cols, dtype=np.int64).reshape(rows, cols)
    u = np.concatenate([idx[:, :-1].ravel(), idx[:-1, :].ravel()])
    v = np.concatenate([idx[:, 1:].ravel(), idx[1:, :].ravel()])
    return csr_from_edges(rows * cols, u, v, name=name or f"lattice_{rows}x{cols}")


def _spatial_order(pts: np.ndarray, cell: float) -> np.ndarray:
    """Row-major cell order of points (locality-preserving ids, as DIMACS rgg)."""
    ncell = max(1, int(math.floor(1.0 / cell)))
    cx = np.minimum((pts[:, 0] * ncell).astype(np.int64), ncell - 1)
    cy = np.minimum((pts[:, 1] * ncell).astype(np.int64), ncell - 1)
    return np.lexsort((pts[:, 0], cx, cy))


def rgg(n: int, radius: Optional[float] = None, seed: int = 1,
        name: Optional[str] = None) -> Graph:
    """Random geometric graph: n uniform points in [0,1]^2, edge iff dist < r.

    r defaults to 0.55*sqrt(ln n / n), which reproduces rgg_n_2_20's m and max
    degree (Table II).
    """
    from scipy.spatial import cKDTree
    if radius is None:
        radius = 0.55 * math.sqrt(math.log(n) / n)
    rng = np.random.default_rng(seed)
    pts = rng.random((n, 2))
    pts = pts[_spatial_order(pts, radius)]
    pairs = cKDTree(pts).query_pairs(radius, output_type="ndarray")
    return csr_from_edges(n, pairs[:, 0], pairs[:, 1], name=name or f"rgg_n{n}")


def delaunay(n: int, seed: int = 1, name: Optional[str] = None) -> Graph:
    """Delaunay triangulation of n uniform points (delaunay_nXX class)."""
    from scipy.spatial import Delaunay
    rng = np.random.default_rng(seed)
    pts = rng.random((n, 2))
    pts = pts[_spatial_order(pts, 1.0 / math.sqrt(n))]
    tri = Delaunay(pts).simplices.astype(np.int64)
    u = np.concatenate([tri[:, 0], tri[:, 1], tri[:, 2]])
    v = np.concatenate([tri[:, 1], tri[:, 2], tri[:, 0]])
    return csr_from_edges(n, u, v, name=name or f"delaunay_n{n}")


def watts_strogatz(n: int, k: int = 10, p: float = 0.2, seed: int = 1,
                   name: Optional[str] = None) -> Graph:
    """Watts-Strogatz small world [37]: ring of k nearest neighbours, each edge
    (u, u+j) rewired with probability p to a uniform random endpoint.

    Rewiring collisions (self-loops, duplicates) are dropped by the CSR builder
    rather than redrawn; k=10, p=0.2 matches Table II 'smallworld'.
    """
    rng = np.random.default_rng(seed)
    base = np.arange(n, dtype=np.int64)
    us, vs = [], []
    for j in range(1, k // 2 + 1):
        v = (base + j) % n
        rew = rng.random(n) < p
        v = np.where(rew, rng.integers(0, n, n), v)
        us.append(base)
        vs.append(v)
    return csr_from_edges(n, np.concatenate(us), np.concatenate(vs),
                          name=name or f"ws_n{n}_k{k}_p{p}")


def path_graph(n: int) -> Graph:
    a = np.arange(n - 1)
    return csr_from_edges(n, a, a + 1, name=f"path{n}")


def star_graph(n: int) -> Graph:
    """Centre 0 with n-1 leaves."""
    return csr_from_edges(n, np.zeros(n - 1, dtype=np.int64), np.arange(1, n), name=f"star{n}")


def cycle_graph(n: int, directed: bool = False) -> Graph:
    a = np.arange(n)
    return csr_from_edges(n, a, (a + 1) % n, directed=directed, name=f"cycle{n}")


def complete_graph(n: int) -> Graph:
    u, v = np.triu_indices(n, 1)
    return csr_from_edges(n, u, v, name=f"K{n}")


def directed_path(n: int) -> Graph:
    a = np.arange(n - 1)
    return csr_from_edges(n, a, a + 1, directed=True, name=f"dpath{n}")


def random_tree(n: int, seed: int = 1) -> Graph:
    rng = np.random.default_rng(seed)
    par = np.array([rng.integers(0, i) for i in range(1, n)], dtype=np.int64)
    return csr_from_edges(n, np.arange(1, n), par, name=f"tree{n}")


def gnp(n: int, p: float, seed: int = 1, directed: bool = False) -> Graph:
    rng = np.random.default_rng(seed)
    if directed:
        mask = rng.random((n, n)) < p
        u, v = np.nonzero(mask)
    else:
        iu, iv = np.triu_indices(n, 1)
        keep = rng.random(iu.size) < p
        u, v = iu[keep], iv[keep]
    return csr_from_edges(n, u, v, directed=directed, name=f"gnp{n}_{p}")


# ------------------------------------------------------------------------ sources


def sample_sources(g: Graph, k: Optional[int], seed: int,
                   exclude_isolated: bool = True) -> np.ndarray:
    """Seeded source list.

    k=None -> all n vertices in id order (exact BC).  Otherwise k distinct
    sources drawn uniformly without replacement from the non-isolated vertices
    (SURVEY.md §8(c) reading #13).
    """
    if k is None:
        return np.arange(g.n, dtype=np.int32)
    pool = np.nonzero(g.degrees() > 0)[0] if exclude_isolated else np.arange(g.n)
    if k > pool.size:
        raise ValueError(f"k={k} > {pool.size} eligible sources")
    rng = np.random.default_rng(seed)
    return np.sort(rng.choice(pool, size=k, replace=False)).astype(np.int32)


def permute_sources(sources: np.ndarray, seed: int) -> np.ndarray:
    """Seeded permutation applied before strided multi-GPU sharding (§8(e))."""
    rng = np.random.default_rng(seed)
    return sources[rng.permutation(sources.size)]


# ------------------------------------------------------------------------ configs


@dataclasses.dataclass
class Config:
    key: str
    description: str
    make: Callable[[], Graph]
    k: Optional[int]          # None = all sources (exact BC)
    seed: int

    def graph(self) -> Graph:
        return self.make()

    def sources(self, g: Graph) -> np.ndarray:
        return sample_sources(g, self.k, self.seed + 7)


CONFIGS: Dict[str, Config] = {
    "c1": Config("c1", "exact BC, all sources, undirected R-MAT scale 10 ef 16",
                 lambda: rmat(10, 16, seed=101, name="rmat_s10_ef16"), None, 101),
    "c2": Config("c2", "exact BC on a 256x256 4-neighbour lattice (2^16 vertices, WE path)",
                 lambda: lattice2d(256, 256), None, 102),
    "c2d": Config("c2d", "exact BC on a Delaunay triangulation of 2^16 points",
                  lambda: delaunay(1 << 16, seed=102), None, 102),
    "c3": Config("c3", "RGG 2^18 vertices, r=0.55*sqrt(ln n/n), 8,192 sampled sources",
                 lambda: rgg(1 << 18, seed=103), 8192, 103),
    "c4": Config("c4", "Graph500 Kronecker scale 18 ef 16, 16,384 sampled sources",
                 lambda: rmat(18, 16, seed=104, name="kron_s18_ef16"), 16384, 104),
    "c5k": Config("c5k", "Graph500 Kronecker scale 22 ef 16, 65,536 sampled sources",
                  lambda: rmat(22, 16, seed=105, name="kron_s22_ef16"), 65536, 105),
    "c5ws": Config("c5ws", "Watts-Strogatz 2^22 vertices k=10 p=0.2, 65,536 sampled sources",
                   lambda: watts_strogatz(1 << 22, 10, 0.2, seed=106), 65536, 106),
}
