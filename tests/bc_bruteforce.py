"""Brute-force references for tiny graphs (test helpers; independent of oracle/).

Eq. (1) evaluated literally: enumerate every simple path between
every ordered pair (s, t) by DFS, keep those of minimal length (the shortest
paths), count sigma_st and sigma_st(v), and sum sigma_st(v)/sigma_st with
exact rationals.  Exponential -- n <= ~9 only.
"""
from __future__ import annotations

from fractions import Fraction
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np


def adjacency(g) -> List[List[int]]:
    ro, col = g.row_offsets, g.col_indices
    return [col[ro[v]:ro[v + 1]].tolist() for v in range(g.n)]


def all_simple_paths(adj, s: int, t: int) -> List[List[int]]:
    out = []
    stack = [(s, [s])]
    while stack:
        v, path = stack.pop()
        if v == t:
            out.append(path)
            continue
        for w in adj[v]:
            if w not in path:
                stack.append((w, path + [w]))
    return out


def shortest_paths(adj, s: int, t: int) -> List[List[int]]:
    paths = all_simple_paths(adj, s, t)
    if not paths:
        return []
    best = min(len(p) for p in paths)
    return [p for p in paths if len(p) == best]


def bc_eq1(g, sources: Optional[Sequence[int]] = None) -> List[Fraction]:
    """BC(v) = h * sum_{s in S} sum_{t != s, t != v} sigma_st(v) / sigma_st (exact)."""
    adj = adjacency(g)
    n = g.n
    S = range(n) if sources is None else sources
    bc = [Fraction(0)] * n
    for s in S:
        for t in range(n):
            if t == s:
                continue
            sp = shortest_paths(adj, s, t)
            if not sp:
                continue
            sigma = len(sp)
            for v in range(n):
                if v == s or v == t:
                    continue
                through = sum(1 for p in sp if v in p)
                if through:
                    bc[v] += Fraction(through, sigma)
    if not g.directed:
        bc = [b / 2 for b in bc]
    return bc


def per_source(g, s: int) -> Tuple[List[int], List[int], List[Fraction]]:
    """d (-1 unreachable), sigma_sv (path counts) and delta_s(v) = sum_t sigma_st(v)/sigma_st."""
    adj = adjacency(g)
    n = g.n
    d = [-1] * n
    sig = [0] * n
    d[s] = 0
    sig[s] = 1
    sps: Dict[int, List[List[int]]] = {}
    for t in range(n):
        if t == s:
            continue
        sp = shortest_paths(adj, s, t)
        sps[t] = sp
        if sp:
            d[t] = len(sp[0]) - 1
            sig[t] = len(sp)
    delta = [Fraction(0)] * n
    for t, sp in sps.items():
        if not sp:
            continue
        for v in range(n):
            if v == s or v == t:
                continue
            through = sum(1 for p in sp if v in p)
            if through:
                delta[v] += Fraction(through, len(sp))
    return d, sig, delta


def to_float(xs) -> np.ndarray:
    return np.array([float(x) for x in xs], dtype=np.float64)
