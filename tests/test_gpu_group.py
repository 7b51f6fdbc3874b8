"""GPU parity of the group engine (BC_ENGINE_GROUP, bc_group.cu) against the CPU oracle.

Same bar as test_gpu_parity.py: d bit-exact, sigma bit-exact below 2^53
(and on the lattice up to 2^505: rows are summed in CSR order by one thread, as in the
oracle), delta and BC within 1e-9.  Group sizes cover the degenerate one-CTA group, odd
sizes (ragged ownership of the hub words), and a single group spanning the whole grid.
"""
import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg

from test_gpu_parity import TWO53, BC_TOL, bcmod, graph, rel_err, check_bc, check_source, small_graphs  # noqa: F401

pytestmark = pytest.mark.gpu

NO_EP = 2147483647  # Alg. 5 guard no frontier reaches: every level work-efficient


def group_graph(bcmod, g, ctas=0, **kw):
    opts = dict(engine="group", group_ctas=ctas)
    opts.update(kw)
    return bcmod.BCGraph.from_graph(g, **opts)


@pytest.mark.parametrize("ctas", [1, 2, 3, 7, 100000])
def test_c1_exact_bc_group_sizes(bcmod, oracle_mod, ctas):
    g = graph("c1")
    with group_graph(bcmod, g, ctas, strategy="we") as bg:
        check_bc(bg, g, None, oracle_mod)
        st = bg.stats()
        assert st["sources"] == g.n and st["ep_levels"] == 0
        assert st["bc_kernel_launches"] == 1


@pytest.mark.parametrize("ctas", [1, 5, 100000])
def test_c1_every_source_d_sigma_delta(bcmod, oracle_mod, ctas):
    g = graph("c1")
    with group_graph(bcmod, g, ctas, strategy="we") as bg:
        for s in range(0, g.n, 3):
            check_source(bg, g, s, oracle_mod)


def test_c1_stats_match_oracle_counters(bcmod, oracle_mod):
    g = graph("c1")
    src = gg.sample_sources(g, 200, seed=3)
    with group_graph(bcmod, g, 4, strategy="we") as bg:
        bg.compute(src)
        st = bg.stats()
    refs = [oracle_mod.single_source(g, int(s)) for s in src]
    assert st["n_reached"] == sum(r["n_reached"] for r in refs)
    assert st["arcs_reached"] == sum(r["arcs_reached"] for r in refs)
    assert st["dag_arcs"] == sum(r["dag_arcs"] for r in refs)
    assert st["levels"] == sum(r["num_levels"] for r in refs)


def test_c2_lattice_sigma_beyond_2p53_bit_exact(bcmod, oracle_mod):
    g = graph("c2")
    with group_graph(bcmod, g, 8, strategy="we") as bg:
        for s in (0, 255, 32896, g.n - 1):
            got, ref = check_source(bg, g, s, oracle_mod)
            assert np.array_equal(got["sigma"], ref["sigma"])  # up to 2^505, every vertex
        src = gg.sample_sources(g, 96, seed=11)
        check_bc(bg, g, src, oracle_mod)


@pytest.mark.parametrize("key,k", [("c2d", 128), ("c3", 64), ("c4", 64)])
def test_subsets(bcmod, oracle_mod, key, k):
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:k] if gg.CONFIGS[key].k else gg.sample_sources(g, k, seed=5)
    with group_graph(bcmod, g, 0, strategy="sampling", ep_min_frontier=NO_EP) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        for s in src[:2]:
            check_source(bg, g, s, oracle_mod)
        st = bg.stats()
        assert st["ep_levels"] == 0 and st["sampling_median"] >= 0


@pytest.mark.parametrize("key", ["c5ws", "c5k"])
@pytest.mark.parametrize("ctas", [0, 37])
def test_c5_subset(bcmod, oracle_mod, key, ctas):
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:32]
    with group_graph(bcmod, g, ctas, strategy="sampling", ep_min_frontier=NO_EP) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        check_source(bg, g, src[0], oracle_mod)


@pytest.mark.parametrize("succ_bits", [-1, 1])
def test_successor_bits_on_off(bcmod, oracle_mod, succ_bits):
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:48]
    with group_graph(bcmod, g, 9, strategy="we", succ_bits=succ_bits) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)


@pytest.mark.parametrize("gi", [0, 1, 2, 3, 4, 5, 10])
@pytest.mark.parametrize("ctas", [1, 3])
def test_edge_case_graphs(bcmod, oracle_mod, gi, ctas):
    g = small_graphs()[gi]  # undirected ones: star, K40, path 700, cycle 513, empty, forest, 1x1
    with group_graph(bcmod, g, ctas, strategy="we") as bg:
        check_bc(bg, g, None, oracle_mod)
        for s in range(min(g.n, 5)):
            check_source(bg, g, s, oracle_mod)


def test_zero_sources_duplicates(bcmod, oracle_mod):
    g = graph("c1")
    with group_graph(bcmod, g, 2, strategy="we") as bg:
        assert np.all(bg.compute(np.zeros(0, dtype=np.int32)) == 0.0)
        src = np.array([5, 5, 17, 5, 900], dtype=np.int32)
        check_bc(bg, g, src, oracle_mod)


def test_directed_and_ep_runs_use_per_source_engine(bcmod, oracle_mod):
    """Launches the group engine cannot run (directed graph, possible EP levels) fall back
    to the per-source engine and stay exact."""
    g = gg.gnp(300, 0.02, seed=3, directed=True)
    with group_graph(bcmod, g, 2, strategy="we") as bg:
        check_bc(bg, g, None, oracle_mod)
    g = graph("c1")
    with group_graph(bcmod, g, 2, strategy="ep") as bg:
        check_bc(bg, g, None, oracle_mod)
        assert bg.stats()["ep_levels"] > 0


def test_sampling_decision_matches_per_source(bcmod, oracle_mod):
    """Alg. 5's sampling phase runs on the group engine too: same keys, same decision."""
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:600]
    res = {}
    for eng in ("per_source", "group"):
        with bcmod.BCGraph.from_graph(g, engine=eng, strategy="sampling", ep_min_frontier=NO_EP) as bg:
            bc = bg.compute(src)
            st = bg.stats()
            res[eng] = (bc, st["sampling_ep"], st["sampling_median"], st["levels"])
    a, b = res["per_source"], res["group"]
    assert a[1:] == b[1:]
    assert rel_err(b[0], a[0]) <= BC_TOL


def test_auto_engine_picks_group_on_large_graphs(bcmod, oracle_mod):
    """Auto engine: group engine on n >= 2^21 when every level is work-efficient (4 groups
    on the unskewed c5ws, groups of 12 CTAs on the relabelled c5k); per-source on c4."""
    for key, groups in (("c5ws", 4), ("c5k", None)):
        g = graph(key)
        src = gg.CONFIGS[key].sources(g)[:24]
        with bcmod.BCGraph.from_graph(g, ep_min_frontier=NO_EP) as bg:
            check_bc(bg, g, src, oracle_mod, nthreads=16)
            st = bg.stats()
            assert st["batches"] == 0 and st["bc_kernel_launches"] == 1
            assert st["inflight"] == groups if groups else 2 <= st["inflight"] <= 64
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:600]
    with bcmod.BCGraph.from_graph(g, ep_min_frontier=NO_EP) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        assert bg.stats()["inflight"] > 64


@pytest.mark.parametrize("key", ["c5ws", "c5k"])
def test_group_matches_per_source_on_many_sources(bcmod, key):
    """Every BFS of 1,024 sources agrees between the engines: the traversal counters (levels,
    reached vertices and arcs, DAG arcs) are exact integers, BC within 1e-9.  Races in the
    group barrier / ownership / bitmap protocol show up here first."""
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:1024]
    out = {}
    for eng in ("per_source", "group"):
        with bcmod.BCGraph.from_graph(g, engine=eng, strategy="we") as bg:
            bc = bg.compute(src)
            st = bg.stats()
            out[eng] = (bc, [st[k] for k in ("levels", "n_reached", "arcs_reached", "dag_arcs")])
    assert out["group"][1] == out["per_source"][1]
    assert rel_err(out["group"][0], out["per_source"][0]) <= BC_TOL


@pytest.mark.parametrize("fast", ["0", "1"])
@pytest.mark.parametrize("key,k", [("c1", None), ("c2", 64), ("c4", 96), ("c5ws", 24), ("c5k", 24)])
def test_generic_and_fast_group_paths(bcmod, oracle_mod, monkeypatch, fast, key, k):
    """The group engine's two implementations of the work-efficient levels -- the generic
    row_pass and the fast path (bc_fast.cuh, G = true; auto on degree-relabelled graphs) --
    on the same graphs, forced with BC_GROUP_FAST: identical d / sigma, BC within 1e-9."""
    monkeypatch.setenv("BC_GROUP_FAST", fast)
    g = graph(key)
    src = None if k is None else (gg.CONFIGS[key].sources(g)[:k] if gg.CONFIGS[key].k
                                   else gg.sample_sources(g, k, seed=6))
    with group_graph(bcmod, g, 0, strategy="we") as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        s0 = 5 if src is None else int(src[0])
        check_source(bg, g, s0, oracle_mod)
        assert bg.stats()["engines"] & 4
