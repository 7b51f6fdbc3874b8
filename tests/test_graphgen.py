"""Generators and CSR builder: structural validity and calibration to Table II
 as measured in SURVEY.md §4.6 / §8(a)."""
import math

import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg


def check_csr(g):
    ro, col = g.row_offsets, g.col_indices
    assert ro.dtype == np.int64 and col.dtype == np.int32
    assert ro[0] == 0 and ro[-1] == col.size and np.all(np.diff(ro) >= 0)
    assert col.size == 0 or (col.min() >= 0 and col.max() < g.n)
    src = np.repeat(np.arange(g.n), g.degrees())
    assert not np.any(src == col), "self-loop"
    key = src.astype(np.int64) * g.n + col
    assert np.all(np.diff(key) > 0), "rows not sorted / duplicate arcs"
    if not g.directed:
        rkey = col.astype(np.int64) * g.n + src
        assert np.array_equal(np.sort(rkey), key), "not symmetric"


def test_csr_builder_dedupe_selfloops():
    g = gg.csr_from_edges(5, np.array([0, 0, 1, 2, 2, 4]), np.array([1, 1, 0, 2, 3, 4]))
    check_csr(g)
    assert g.m == 2 and g.nnz == 4
    assert g.degrees().tolist() == [1, 1, 1, 1, 0]
    d = gg.csr_from_edges(3, np.array([0, 1]), np.array([1, 2]), directed=True)
    check_csr(d)
    assert d.m == 2 and d.degrees().tolist() == [1, 1, 0]
    with pytest.raises(ValueError):
        gg.csr_from_edges(3, np.array([0]), np.array([3]))


@pytest.mark.parametrize("make", [
    lambda: gg.rmat(10, 16, seed=101), lambda: gg.lattice2d(7, 5), lambda: gg.rgg(3000, seed=1),
    lambda: gg.delaunay(2000, seed=2), lambda: gg.watts_strogatz(1000, 10, 0.2, seed=3),
    lambda: gg.gnp(100, 0.05, seed=4, directed=True), lambda: gg.random_tree(50),
])
def test_generators_valid(make):
    check_csr(make())


def test_generators_seeded():
    a, b = gg.rmat(9, 16, seed=5), gg.rmat(9, 16, seed=5)
    assert np.array_equal(a.col_indices, b.col_indices)
    c = gg.rmat(9, 16, seed=6)
    assert not np.array_equal(a.col_indices, c.col_indices)


def test_c1_rmat_calibration():
    g = gg.CONFIGS["c1"].graph()
    assert g.n == 1024
    assert 10000 < g.m < 11000          # m ~ 10.5k
    iso = int((g.degrees() == 0).sum())
    assert 100 < iso < 200              # ~145 isolated


def test_lattice_counts():
    g = gg.lattice2d(256, 256)
    assert g.n == 65536 and g.m == 130560 and g.degrees().max() == 4


def test_smallworld_calibration():
    """Table II smallworld: n=100,000, m=499,998, max degree 17."""
    g = gg.watts_strogatz(100_000, 10, 0.2, seed=1)
    assert abs(g.m - 499_998) / 499_998 < 0.001
    assert 15 <= g.degrees().max() <= 19


def test_rgg_calibration():
    """r = 0.55 sqrt(ln n / n) reproduces rgg_n_2_20's m/n ratio (6,891,620 / 2^20)."""
    n = 1 << 16
    g = gg.rgg(n, seed=3)
    want = 6_891_620 / (1 << 20) * n * (math.log(n) / math.log(1 << 20))
    assert abs(g.m - want) / want < 0.03


def test_delaunay_m_about_3n():
    n = 1 << 14
    g = gg.delaunay(n, seed=4)
    assert 3 * n - 6 * math.isqrt(n) < g.m <= 3 * n - 6


def test_sources():
    g = gg.rmat(10, 16, seed=101)
    s = gg.sample_sources(g, 300, seed=1)
    assert s.dtype == np.int32 and len(np.unique(s)) == 300
    assert np.all(g.degrees()[s] > 0)
    assert np.array_equal(gg.sample_sources(g, None, 0), np.arange(g.n))
    p = gg.permute_sources(s, 2)
    assert np.array_equal(np.sort(p), s)


@pytest.mark.parametrize("directed", [False, True])
def test_native_csr_builder_matches_numpy_reference(directed):
    n, u, v = gg.rmat_edges(11, 16, seed=9)
    u = np.concatenate([u, [3, 5]])          # explicit self-loop and duplicate
    v = np.concatenate([v, [3, int(v[0])]])
    u[-1] = u[0]
    a = gg.csr_from_edges(n, u, v, directed=directed)
    b = gg.csr_from_edges_numpy(n, u, v, directed=directed)
    assert np.array_equal(a.row_offsets, b.row_offsets)
    assert np.array_equal(a.col_indices, b.col_indices)
    check_csr(a)
    with pytest.raises(ValueError):
        gg.csr_from_edges(4, np.array([0]), np.array([4]))


def test_rmat_edges_are_counter_based():
    """Edge i depends only on (seed, i): a longer draw extends a shorter one."""
    _, u1, v1 = gg.rmat_edges(8, 4, seed=3, relabel=False)
    _, u2, v2 = gg.rmat_edges(8, 8, seed=3, relabel=False)
    assert np.array_equal(u1, u2[:u1.size]) and np.array_equal(v1, v2[:v1.size])


def test_kron_s22_calibration_numbers():
    """m ~ 64.15M, ~42.9 % isolated, max degree ~163k (seeded draw)."""
    g = gg.CONFIGS["c5k"].graph()
    d = g.degrees()
    assert abs(g.m - 64.15e6) / 64.15e6 < 0.01
    assert 0.40 < (d == 0).mean() < 0.46
    assert 100_000 < d.max() < 250_000
