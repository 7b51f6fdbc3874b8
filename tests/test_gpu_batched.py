"""GPU parity of the multi-source batched engine (BC_ENGINE_BATCHED)
against the CPU oracle, through the C ABI.

Same bar as tests/test_gpu_parity.py: d bit-exact; sigma bit-exact wherever the
oracle's sigma is below 2^53 (rows are pulled in CSR order, the oracle's order), within
1e-12 relative above; delta and BC within 1e-9 (|gpu - ref| / max(|ref|, 1)).
Batches of 64 sources: full batches, ragged tails (k mod 64 != 0), duplicates, rows
split across many warp ranges (hub_chunk small), batches deeper than the level cap
(rerun per source), and the auto engine's choice (Alg. 5 EP run on a large skewed graph).
"""
import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg

pytestmark = pytest.mark.gpu

TWO53 = 2.0 ** 53
BC_TOL = 1e-9


@pytest.fixture(scope="module")
def bcmod():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    bcm.load_library()
    return bcm


_graphs = {}


def graph(key):
    if key not in _graphs:
        _graphs[key] = gg.CONFIGS[key].graph()
    return _graphs[key]


def rel_err(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    if a.size == 0:
        return 0.0
    return float(np.max(np.abs(a - b) / np.maximum(np.abs(b), 1.0)))


def check_batch(bg, g, sources, oracle_mod):
    got = bg.batch_sources(sources)
    for b, s in enumerate(sources):
        ref = oracle_mod.single_source(g, int(s))
        assert np.array_equal(got["d"][b], ref["d"]), f"d mismatch, source {s} (slot {b})"
        small = ref["sigma"] < TWO53
        assert np.array_equal(got["sigma"][b][small], ref["sigma"][small]), f"sigma mismatch, source {s}"
        assert rel_err(got["sigma"][b], ref["sigma"]) < 1e-12
        assert rel_err(got["delta"][b], ref["delta"]) < BC_TOL, f"delta, source {s}"
    return got


def check_bc(bg, g, sources, oracle_mod, nthreads=8):
    got = bg.compute(sources)
    ref = oracle_mod.bc(g, sources, nthreads=nthreads)
    err = rel_err(got, ref)
    assert err <= BC_TOL, f"BC max rel err {err}"
    return got, ref


# ------------------------------------------------------------------ C1 (R-MAT s10)


def test_c1_batched_exact_bc(bcmod, oracle_mod):
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we") as bg:
        check_bc(bg, g, None, oracle_mod)
        st = bg.stats()
        assert st["sources"] == g.n
        assert st["batches"] == (g.n + 63) // 64 and st["batch_overflows"] == 0


def test_c1_batch_d_sigma_delta(bcmod, oracle_mod):
    g = graph("c1")
    rng = np.random.default_rng(5)
    with bcmod.BCGraph.from_graph(g, engine="batched") as bg:
        check_batch(bg, g, np.arange(64, dtype=np.int32), oracle_mod)           # full batch
        check_batch(bg, g, rng.choice(g.n, 37, replace=False).astype(np.int32), oracle_mod)  # ragged
        check_batch(bg, g, np.array([7], dtype=np.int32), oracle_mod)          # single source
        dup = np.array([3, 3, 900, 3, 1023, 0], dtype=np.int32)               # duplicates
        check_batch(bg, g, dup, oracle_mod)
        iso = np.flatnonzero(g.degrees() == 0)
        if iso.size:
            check_batch(bg, g, np.array([iso[0], 5, iso[-1]], dtype=np.int32), oracle_mod)


def test_c1_batched_stats_match_oracle_counters(bcmod, oracle_mod):
    g = graph("c1")
    src = gg.sample_sources(g, 200, seed=3)
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we") as bg:
        bg.compute(src)
        st = bg.stats()
    refs = [oracle_mod.single_source(g, int(s)) for s in src]
    assert st["sources"] == src.size
    assert st["n_reached"] == sum(r["n_reached"] for r in refs)
    assert st["arcs_reached"] == sum(r["arcs_reached"] for r in refs)
    assert st["dag_arcs"] == sum(r["dag_arcs"] for r in refs)
    assert st["levels"] == sum(r["num_levels"] for r in refs)


@pytest.mark.parametrize("chunk", [4, 33, 200])
def test_c1_hub_chunks(bcmod, oracle_mod, chunk):
    """hub_chunk = minimum arcs per warp range: tiny ranges split every row over many
    warps, whose fp64 reductions meet in the row's accumulators."""
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we", hub_chunk=chunk) as bg:
        check_bc(bg, g, None, oracle_mod)
        hubs = np.argsort(-g.degrees())[:40].astype(np.int32)  # hub sources: level-0 chunks
        check_batch(bg, g, hubs, oracle_mod)


def test_sources_subset_and_order(bcmod, oracle_mod):
    g = graph("c1")
    rng = np.random.default_rng(11)
    src = rng.integers(0, g.n, 301).astype(np.int32)  # duplicates, ragged last batch
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we") as bg:
        a, _ = check_bc(bg, g, src, oracle_mod)
        b = bg.compute(src[::-1].copy())
        assert rel_err(a, b) < 1e-12
        z = bg.compute(np.zeros(0, dtype=np.int32))
        assert not z.any()


# --------------------------------------------------------- level cap / overflow


def test_overflow_rerun_per_source(bcmod, oracle_mod):
    """A 40x40 lattice has depth up to 78: with batch_levels=16 most batches overflow and
    are rerun by the per-source kernel; the BC is unchanged."""
    g = gg.lattice2d(40, 40)
    rng = np.random.default_rng(2)
    src = rng.choice(g.n, 150, replace=False).astype(np.int32)
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we", batch_levels=16) as bg:
        check_bc(bg, g, src, oracle_mod)
        st = bg.stats()
        assert st["batch_overflows"] > 0 and st["sources"] == src.size
        with pytest.raises(bcmod.BCError):
            bg.batch_sources(np.array([0], dtype=np.int32))  # corner: depth 78 > 16
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we", batch_levels=100) as bg:
        check_bc(bg, g, src, oracle_mod)
        assert bg.stats()["batch_overflows"] == 0
        # sigma up to C(78, 39) ~ 2^74: <= 2 predecessors per vertex, so any order is exact
        got = bg.batch_sources(np.array([0, 1599, 820], dtype=np.int32))
        for b, s in enumerate((0, 1599, 820)):
            ref = oracle_mod.single_source(g, s)
            assert np.array_equal(got["sigma"][b], ref["sigma"])
            assert np.array_equal(got["d"][b], ref["d"])


def test_delaunay_batched_sigma_above_2p53(bcmod, oracle_mod):
    g = graph("c2d")  # depth ~100-117, sigma up to ~2^53.4
    rng = np.random.default_rng(4)
    src = rng.choice(g.n, 64, replace=False).astype(np.int32)
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we", batch_levels=200) as bg:
        check_batch(bg, g, src[:16], oracle_mod)
        check_bc(bg, g, src, oracle_mod)


# ----------------------------------------------------------------- auto engine


def test_auto_engine_follows_alg5(bcmod, oracle_mod):
    """Auto: batched only for an Alg. 5 EP run on a large skewed graph (c5k); c4 and the
    high-diameter lattice stay per source."""
    g = graph("c5k")
    src = gg.sample_sources(g, 512 + 128, seed=9)
    with bcmod.BCGraph.from_graph(g) as bg:  # defaults: sampling, auto engine
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        st = bg.stats()
        assert st["sampling_ep"] == 1 and st["batches"] == 2
        assert st["sources"] == src.size
    g4 = graph("c4")
    src4 = gg.sample_sources(g4, 512 + 64, seed=9)
    with bcmod.BCGraph.from_graph(g4) as bg:
        check_bc(bg, g4, src4, oracle_mod, nthreads=16)
        st = bg.stats()
        assert st["sampling_ep"] == 1 and st["batches"] == 0
    g2 = gg.lattice2d(64, 64)  # high diameter: Alg. 5 -> WE -> per-source engine
    with bcmod.BCGraph.from_graph(g2) as bg:
        src2 = np.arange(0, g2.n, 7, dtype=np.int32)
        check_bc(bg, g2, src2, oracle_mod)
        st = bg.stats()
        assert st["sampling_ep"] == 0 and st["batches"] == 0


def test_c5ws_batched_subset(bcmod, oracle_mod):
    g = graph("c5ws")
    src = gg.sample_sources(g, 128, seed=17)
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we") as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        check_batch(bg, g, src[:4], oracle_mod)


def test_c5k_batched_subset(bcmod, oracle_mod):
    g = graph("c5k")
    src = gg.sample_sources(g, 128, seed=19)
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we") as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        st = bg.stats()
        assert st["batch_overflows"] == 0


def test_graphs_without_edges(bcmod):
    g = gg.csr_from_edges(5, np.zeros(0, np.int64), np.zeros(0, np.int64))
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy="we") as bg:
        assert not bg.compute(None).any()
        out = bg.batch_sources(np.array([0, 4], dtype=np.int32))
        assert out["d"][0, 0] == 0 and (out["d"][0, 1:] == -1).all()


def test_directed_rejected(bcmod):
    g = gg.directed_path(6)
    with bcmod.BCGraph.from_graph(g, engine="batched") as bg:
        with pytest.raises(bcmod.BCError):
            bg.batch_sources(np.array([0], dtype=np.int32))


@pytest.mark.parametrize("key,k,strategy", [("c1", None, "ep"), ("c1", 600, "sampling"), ("c4", 200, "ep"),
                                            ("c4", 700, "sampling"), ("c5k", 640, "sampling")])
def test_multi_source_ep_levels(bcmod, oracle_mod, key, k, strategy):
    """Multi-source edge-parallel levels: one scan of all arcs serves the
    64 sources of a batch when the union frontier reaches the Alg. 5 guard (strategy
    sampling, after an EP decision) or on every level (strategy ep).  BC, the per-source
    d / sigma / delta of a batch and the byte-model counters equal the oracle's."""
    g = graph(key)
    src = None if k is None else gg.CONFIGS[key].sources(g)[:k] if gg.CONFIGS[key].k \
        else gg.sample_sources(g, k, seed=13)
    with bcmod.BCGraph.from_graph(g, engine="batched", strategy=strategy) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        st = bg.stats()
        assert st["ep_levels"] > 0 and st["batches"] > 0
        if strategy == "ep":
            assert st["we_levels"] == 0
        else:
            assert st["sampling_ep"] == 1
        sub = (np.arange(g.n, dtype=np.int32) if src is None else src)[:40]
        check_batch(bg, g, sub, oracle_mod)   # the last call's Alg. 5 decision stands (EP)
    if key != "c5k":
        refs = [oracle_mod.single_source(g, int(s)) for s in (np.arange(g.n) if src is None else src)]
        assert st["n_reached"] == sum(r["n_reached"] for r in refs)
        assert st["arcs_reached"] == sum(r["arcs_reached"] for r in refs)
        assert st["dag_arcs"] == sum(r["dag_arcs"] for r in refs)
        assert st["levels"] == sum(r["num_levels"] for r in refs)
        assert st["dist_sum"] == sum(int(r["d"][r["d"] >= 0].sum()) for r in refs)
