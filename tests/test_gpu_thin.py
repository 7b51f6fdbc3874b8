"""GPU parity of the group engine's thin-row passes (bc_thin.cuh: one row per virtual warp
of a few lanes) against the CPU oracle, forced with BC_GROUP_MODE=2 on every
graph kind (auto picks them for large graphs without hubs: c5ws).

Same bar as test_gpu_parity.py: d bit-exact, sigma bit-exact below 2^53,
delta and BC within 1e-9.  The virtual-warp sums are not in CSR order, so sigma above 2^53
(the lattice) is only checked to 1e-12.  Rows longer than THIN_MAX_ROW (star centre, K40,
Kronecker hubs) take the queued one-warp path; the 1,500-vertex path goes past the group
kernel's RCAP levels (backward levels cut over the whole group).
"""
import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg

from test_gpu_parity import BC_TOL, bcmod, graph, rel_err, check_bc, check_source, small_graphs  # noqa: F401

pytestmark = pytest.mark.gpu

NO_EP = 2147483647


@pytest.fixture
def thin(monkeypatch):
    monkeypatch.setenv("BC_GROUP_MODE", "2")
    monkeypatch.delenv("BC_GROUP_FAST", raising=False)


def thin_graph(bcmod, g, ctas=0, **kw):
    opts = dict(engine="group", group_ctas=ctas, strategy="we")
    opts.update(kw)
    return bcmod.BCGraph.from_graph(g, **opts)


@pytest.mark.parametrize("ctas", [1, 3, 37, 100000])
def test_c1_exact_bc(bcmod, oracle_mod, thin, ctas):
    g = graph("c1")
    with thin_graph(bcmod, g, ctas) as bg:
        check_bc(bg, g, None, oracle_mod)
        for s in range(0, g.n, 97):
            check_source(bg, g, s, oracle_mod)
        st = bg.stats()
        assert st["sources"] == g.n and st["engines"] & 4


def test_c1_counters_match_oracle(bcmod, oracle_mod, thin):
    g = graph("c1")
    src = gg.sample_sources(g, 200, seed=3)
    with thin_graph(bcmod, g, 4) as bg:
        bg.compute(src)
        st = bg.stats()
    refs = [oracle_mod.single_source(g, int(s)) for s in src]
    for k, rk in (("n_reached", "n_reached"), ("arcs_reached", "arcs_reached"), ("dag_arcs", "dag_arcs"),
                  ("levels", "num_levels")):
        assert st[k] == sum(r[rk] for r in refs), k


@pytest.mark.parametrize("key,k", [("c2", 48), ("c2d", 96), ("c3", 64), ("c4", 64)])
def test_subsets(bcmod, oracle_mod, thin, key, k):
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:k] if gg.CONFIGS[key].k else gg.sample_sources(g, k, seed=5)
    with thin_graph(bcmod, g, 0, strategy="sampling", ep_min_frontier=NO_EP) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        for s in src[:2]:
            check_source(bg, g, s, oracle_mod)


@pytest.mark.parametrize("key", ["c5ws", "c5k"])
@pytest.mark.parametrize("ctas", [0, 37])
def test_c5_subset(bcmod, oracle_mod, thin, key, ctas):
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:32]
    with thin_graph(bcmod, g, ctas) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        check_source(bg, g, src[0], oracle_mod)


@pytest.mark.parametrize("gi", [0, 1, 2, 3, 4, 5, 10])
@pytest.mark.parametrize("ctas", [1, 3])
def test_edge_case_graphs(bcmod, oracle_mod, thin, gi, ctas):
    g = small_graphs()[gi]  # star (hub row > THIN_MAX_ROW), K40, path 700, cycle 513, empty, forest, 1x1
    with thin_graph(bcmod, g, ctas) as bg:
        check_bc(bg, g, None, oracle_mod)
        for s in range(min(g.n, 5)):
            check_source(bg, g, s, oracle_mod)


def test_long_path_past_rcap(bcmod, oracle_mod, thin):
    g = gg.path_graph(1500)
    with thin_graph(bcmod, g, 3) as bg:
        check_bc(bg, g, np.array([0, 1499, 700], dtype=np.int32), oracle_mod)
        check_source(bg, g, 0, oracle_mod)


@pytest.mark.parametrize("key", ["c5ws"])
def test_thin_matches_per_source_on_many_sources(bcmod, thin, key):
    """1,024 c5ws sources: integer traversal counters identical to the per-source engine,
    BC within 1e-9 (races in the thin passes' marks or successor windows show up here)."""
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


def test_auto_picks_thin_rows_on_c5ws(bcmod, oracle_mod, monkeypatch):
    """Auto engine on c5ws (2^22 vertices, no hubs, own order): group engine with thin rows;
    on c5k (degree-relabelled) the fast path."""
    monkeypatch.delenv("BC_GROUP_MODE", raising=False)
    monkeypatch.delenv("BC_GROUP_FAST", raising=False)
    for key, mode in (("c5ws", 2), ("c5k", 1)):
        g = graph(key)
        src = gg.CONFIGS[key].sources(g)[:16]
        with bcmod.BCGraph.from_graph(g, ep_min_frontier=NO_EP) as bg:
            check_bc(bg, g, src, oracle_mod, nthreads=16)
            st = bg.stats()
            assert st["engines"] == 4 and st["group_mode"] == mode
