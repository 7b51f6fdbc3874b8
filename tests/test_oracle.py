"""Pins for the CPU oracle (oracle/), against things other than itself.

Each test names what fixes the expected value: Eq. (1) brute force with exact
rationals, closed forms, the sum-of-distances invariant, scipy BFS distances,
lattice binomials, networkx (a library routine), and agreement between the
oracle's two independently written variants (pull vs textbook push).
"""
from math import comb

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components, shortest_path

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
import bc_bruteforce as bf

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")


def scipy_dist(g, sources):
    A = sp.csr_matrix((np.ones(g.nnz), g.col_indices, g.row_offsets), shape=(g.n, g.n))
    D = shortest_path(A, directed=g.directed, unweighted=True, indices=np.asarray(sources))
    D = np.where(np.isinf(D), -1, D).astype(np.int64)
    return D


def rel_err(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    return float(np.max(np.abs(a - b) / np.maximum(np.abs(b), 1.0))) if a.size else 0.0


TINY = [
    gg.gnp(7, 0.45, seed=1), gg.gnp(8, 0.35, seed=2), gg.gnp(8, 0.5, seed=3),
    gg.gnp(9, 0.3, seed=4), gg.cycle_graph(6), gg.lattice2d(3, 3),
    gg.gnp(7, 0.3, seed=5, directed=True), gg.gnp(8, 0.25, seed=6, directed=True),
    gg.csr_from_edges(8, np.array([0, 1, 2, 4, 5]), np.array([1, 2, 0, 5, 6])),  # 2 comps + isolated
]


@pytest.mark.parametrize("gi", range(len(TINY)))
def test_bc_equals_eq1_bruteforce(oracle_mod, gi):
    g = TINY[gi]
    exact = bf.to_float(bf.bc_eq1(g))
    assert rel_err(oracle_mod.bc(g), exact) < 1e-13
    assert rel_err(oracle_mod.bc_push(g), exact) < 1e-13


@pytest.mark.parametrize("gi", [0, 2, 6])
def test_subset_bc_equals_eq1_bruteforce(oracle_mod, gi):
    g = TINY[gi]
    S = [1, 4, 4, 6]  # duplicates count with multiplicity
    exact = bf.to_float(bf.bc_eq1(g, S))
    assert rel_err(oracle_mod.bc(g, np.array(S)), exact) < 1e-13


@pytest.mark.parametrize("gi", range(len(TINY)))
def test_single_source_equals_bruteforce(oracle_mod, gi):
    g = TINY[gi]
    for s in range(g.n):
        d, sig, delta = bf.per_source(g, s)
        r = oracle_mod.single_source(g, s)
        assert r["d"].tolist() == d
        assert r["sigma"].tolist() == [float(x) for x in sig]
        assert rel_err(r["delta"], bf.to_float(delta)) < 1e-13


# ------------------------------------------------------------- closed forms


def test_path_closed_form(oracle_mod):
    for n in (2, 3, 9, 50):
        g = gg.path_graph(n)
        i = np.arange(n)
        assert np.array_equal(oracle_mod.bc(g), (i * (n - 1 - i)).astype(float))


def test_star_closed_form(oracle_mod):
    for n in (3, 9, 40):
        b = oracle_mod.bc(gg.star_graph(n))
        assert b[0] == (n - 1) * (n - 2) / 2 and np.all(b[1:] == 0)


def test_cycle_closed_form(oracle_mod):
    for n in (5, 7, 8, 12, 31):
        want = (n - 1) * (n - 3) / 8 if n % 2 else (n - 2) ** 2 / 8
        assert rel_err(oracle_mod.bc(gg.cycle_graph(n)), np.full(n, want)) < 1e-14


def test_complete_graph_zero(oracle_mod):
    assert np.all(oracle_mod.bc(gg.complete_graph(9)) == 0)


def test_directed_path_and_cycle(oracle_mod):
    n = 9
    i = np.arange(n)
    assert np.array_equal(oracle_mod.bc(gg.directed_path(n)), (i * (n - 1 - i)).astype(float))
    b = oracle_mod.bc(gg.cycle_graph(n, directed=True))
    assert np.all(b == (n - 1) * (n - 2) / 2)


def test_tree_closed_form(oracle_mod):
    """Trees: sigma == 1 and BC(v) = sum_{i<j} c_i c_j over component sizes of T - v."""
    g = gg.random_tree(60, seed=3)
    b = oracle_mod.bc(g)
    A = sp.csr_matrix((np.ones(g.nnz), g.col_indices, g.row_offsets), shape=(g.n, g.n)).tolil()
    for v in range(g.n):
        B = A.copy()
        B[v, :] = 0
        B[:, v] = 0
        _, lab = connected_components(B.tocsr(), directed=False)
        sizes = np.bincount(np.delete(lab, v))
        want = (sizes.sum() ** 2 - (sizes ** 2).sum()) / 2
        assert b[v] == want
    r = oracle_mod.single_source(g, 7)
    assert np.all(r["sigma"] == 1.0)


def test_lattice_d_and_sigma_closed_form(oracle_mod):
    """4-neighbour lattice: d = Manhattan distance, sigma = C(|dx|+|dy|, |dx|)."""
    R = C = 64
    g = gg.lattice2d(R, C)
    for s in (0, 31 * C + 17, R * C - 1):
        r = oracle_mod.single_source(g, s)
        sy, sx = divmod(s, C)
        y, x = np.divmod(np.arange(g.n), C)
        dx, dy = np.abs(x - sx), np.abs(y - sy)
        assert np.array_equal(r["d"], dx + dy)
        exact = [comb(int(a + b), int(a)) for a, b in zip(dx, dy)]
        for v, e in enumerate(exact):
            if e < 2 ** 53:
                assert r["sigma"][v] == float(e)
            else:
                assert abs(r["sigma"][v] - e) / e < 1e-12


# ---------------------------------------------------------------- invariant


@pytest.mark.parametrize("make", [
    lambda: gg.watts_strogatz(300, 6, 0.2, seed=1),
    lambda: gg.rmat(9, 8, seed=2),
    lambda: gg.gnp(150, 0.03, seed=3, directed=True),
    lambda: gg.lattice2d(20, 15),
])
def test_sum_of_distances_invariant(oracle_mod, make):
    """sum_v BC(v) = h * sum_{s in S} sum_{t reachable, t != s} (d(s,t) - 1)."""
    g = make()
    rng = np.random.default_rng(0)
    for S in (None, rng.choice(g.n, 25, replace=False)):
        src = np.arange(g.n) if S is None else S
        D = scipy_dist(g, src)
        h = 1.0 if g.directed else 0.5
        want = h * float(np.where(D > 0, D - 1, 0).sum())
        got = oracle_mod.bc(g, None if S is None else S.astype(np.int32)).sum()
        assert abs(got - want) <= 1e-9 * max(1.0, want)


def test_distances_and_levels_vs_scipy(oracle_mod):
    for g in (gg.rmat(11, 16, seed=5), gg.rgg(4000, seed=6), gg.delaunay(3000, seed=7),
              gg.gnp(300, 0.01, seed=8, directed=True)):
        srcs = np.random.default_rng(1).choice(g.n, 6, replace=False)
        D = scipy_dist(g, srcs)
        deg = g.degrees()
        for s, drow in zip(srcs, D):
            r = oracle_mod.single_source(g, int(s))
            assert np.array_equal(r["d"], drow)
            reach = drow >= 0
            assert np.array_equal(r["level_sizes"], np.bincount(drow[reach]))
            assert r["n_reached"] == reach.sum()
            assert r["arcs_reached"] == deg[reach].sum()
            src = np.repeat(np.arange(g.n), deg)
            dsrc, ddst = drow[src], drow[g.col_indices]
            assert r["dag_arcs"] == int(((dsrc >= 0) & (ddst == dsrc + 1)).sum())


# ----------------------------------------------------------------- networkx


def to_nx(g):
    import networkx as nx
    G = nx.DiGraph() if g.directed else nx.Graph()
    G.add_nodes_from(range(g.n))
    src = np.repeat(np.arange(g.n), g.degrees())
    G.add_edges_from(zip(src.tolist(), g.col_indices.tolist()))
    return G


@pytest.mark.parametrize("make", [
    lambda: gg.rmat(10, 16, seed=101),
    lambda: gg.watts_strogatz(1500, 10, 0.2, seed=2),
    lambda: gg.gnp(200, 0.02, seed=3, directed=True),
    lambda: gg.delaunay(1200, seed=4),
])
def test_vs_networkx(oracle_mod, make):
    import networkx as nx
    g = make()
    G = to_nx(g)
    ref = nx.betweenness_centrality(G, normalized=False)
    assert rel_err(oracle_mod.bc(g, nthreads=4), [ref[i] for i in range(g.n)]) < 1e-12
    S = np.random.default_rng(2).choice(g.n, 40, replace=False)
    refs = nx.betweenness_centrality_subset(G, sources=S.tolist(), targets=list(range(g.n)),
                                            normalized=False)
    # networkx halves subset scores for undirected graphs, as the paper does
    assert rel_err(oracle_mod.bc(g, S.astype(np.int32)), [refs[i] for i in range(g.n)]) < 1e-12


# ------------------------------------------------------- push vs pull variants


def test_pull_and_push_variants_agree(oracle_mod):
    for g in (gg.rgg(20000, seed=9), gg.rmat(12, 16, seed=10), gg.lattice2d(90, 90)):
        for s in np.random.default_rng(3).choice(g.n, 4, replace=False):
            a = oracle_mod.single_source(g, int(s))
            b = oracle_mod.single_source_push(g, int(s))
            assert np.array_equal(a["d"], b["d"])
            small = a["sigma"] < 2.0 ** 53
            assert np.array_equal(a["sigma"][small], b["sigma"][small])
            assert rel_err(a["sigma"], b["sigma"]) < 1e-12
            keep = np.arange(g.n) != s  # push accumulates delta_s(s) too; Alg. 3 skips depth 0
            assert rel_err(a["delta"][keep], b["delta"][keep]) < 1e-10


def test_invalid_inputs(oracle_mod):
    g = gg.path_graph(4)
    with pytest.raises(ValueError):
        oracle_mod.bc(g, np.array([5], dtype=np.int32))
    with pytest.raises(ValueError):
        oracle_mod.single_source(g, -1)


def test_empty_and_isolated(oracle_mod):
    g = gg.csr_from_edges(5, np.array([], dtype=np.int64), np.array([], dtype=np.int64))
    assert np.all(oracle_mod.bc(g) == 0)
    r = oracle_mod.single_source(g, 2)
    assert r["num_levels"] == 1 and r["n_reached"] == 1
    assert np.all(oracle_mod.bc(gg.path_graph(5), np.zeros(0, dtype=np.int32)) == 0)


# ------------------------------------------------------------- golden fixtures


def test_fig1_consistent_golden(oracle_mod):
    """tests/golden/fig1_consistent.txt: hand-derived Eq. (1) values on a graph that
    satisfies the Figure 1 prose."""
    import golden_io
    g, want = golden_io.load("fig1_consistent.txt")
    got = oracle_mod.bc(g)
    assert np.array_equal(got, want)
    # the prose itself: 4 (index 3) scores highest; 8 and 9 score zero
    assert int(np.argmax(got)) == 3 and got[7] == 0 and got[8] == 0
    # BFS from 4 has second frontier {1, 3, 5, 6}; 5 -> 9 is 5-7-9
    r4 = oracle_mod.single_source(g, 3)
    assert sorted(np.flatnonzero(r4["d"] == 1) + 1) == [1, 3, 5, 6]
    r5 = oracle_mod.single_source(g, 4)
    assert r5["d"][8] == 2 and r5["sigma"][8] == 1 and r5["d"][6] == 1
