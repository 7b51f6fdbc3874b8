"""GPU parity of the pushed backward levels (bc_fast.cuh push_level / push_rows):
a backward level L whose next level's rows hold fewer arcs (bpush * A_{L+1} < A_L) is
finished from dependencies PUSHED by the level-(L+1) vertices (fp64 atomics into an
accumulator), instead of pulled over level L's own rows (Alg. 3).  Same bar as
test_gpu_parity.py: d bit-exact, sigma bit-exact below 2^53, delta and BC within 1e-9.
BC_BPUSH sets the ratio (0 = always pull, 1 = push whenever the next level is smaller).
"""
import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg

from test_gpu_parity import BC_TOL, bcmod, graph, rel_err, check_bc, check_source, small_graphs  # noqa: F401

pytestmark = pytest.mark.gpu

NO_EP = 2147483647


@pytest.mark.parametrize("ratio", ["1", "4"])
def test_c1_exact_bc(bcmod, oracle_mod, monkeypatch, ratio):
    monkeypatch.setenv("BC_BPUSH", ratio)
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g, strategy="we") as bg:
        check_bc(bg, g, None, oracle_mod)
        for s in range(0, g.n, 61):
            check_source(bg, g, s, oracle_mod)


@pytest.mark.parametrize("key,k", [("c2d", 64), ("c3", 64), ("c4", 256)])
def test_subsets_bench_options(bcmod, oracle_mod, monkeypatch, key, k):
    monkeypatch.setenv("BC_BPUSH", "1")
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:k] if gg.CONFIGS[key].k else gg.sample_sources(g, k, seed=5)
    with bcmod.BCGraph.from_graph(g, strategy="sampling", ep_min_frontier=NO_EP) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        for s in src[:3]:
            check_source(bg, g, s, oracle_mod)


def test_push_scans_fewer_arcs_on_kronecker(bcmod, monkeypatch):
    """On the Kronecker graph the big middle level's rows hold most arcs: pushing its
    dependencies from the next level scans fewer arcs, with the same BC (1e-9)."""
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:512]
    out = {}
    for ratio in ("0", "2"):
        monkeypatch.setenv("BC_BPUSH", ratio)
        with bcmod.BCGraph.from_graph(g, strategy="sampling", ep_min_frontier=NO_EP) as bg:
            bc = bg.compute(src)
            st = bg.stats()
            out[ratio] = (bc, st["arcs_scanned"], st["arcs_reached"], st["dag_arcs"])
    assert out["0"][2:] == out["2"][2:]
    assert out["2"][1] < 0.8 * out["0"][1]
    assert rel_err(out["2"][0], out["0"][0]) <= BC_TOL


@pytest.mark.parametrize("gi", [0, 1, 2, 3, 5, 10])
def test_edge_case_graphs(bcmod, oracle_mod, monkeypatch, gi):
    monkeypatch.setenv("BC_BPUSH", "1")
    g = small_graphs()[gi]  # star, K40, path 700, cycle 513, forest, 1x1
    with bcmod.BCGraph.from_graph(g, strategy="we") as bg:
        check_bc(bg, g, None, oracle_mod)
        for s in range(min(g.n, 5)):
            check_source(bg, g, s, oracle_mod)


@pytest.mark.parametrize("key,k", [("c4", 96), ("c5k", 24)])
def test_group_fast_path_push(bcmod, oracle_mod, monkeypatch, key, k):
    """Group engine, fast path (auto on degree-relabelled graphs): pushed levels across the
    CTAs of a group (owners push, group barrier, owners finish)."""
    monkeypatch.setenv("BC_BPUSH", "1")
    monkeypatch.setenv("BC_GROUP_MODE", "1")
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:k]
    with bcmod.BCGraph.from_graph(g, engine="group", strategy="we") as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        check_source(bg, g, src[0], oracle_mod)
        st = bg.stats()
        assert st["engines"] == 4 and st["group_mode"] == 1
