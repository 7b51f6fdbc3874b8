"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar: d bit-exact; sigma bit-exact wherever the oracle's sigma is
below 2^53, within 1e-12 relative above; delta and BC within max relative error
1e-9 (|gpu - ref| / max(|ref|, 1)).  Sizes span several 256-vertex tiles and
ragged tails; the full-size bench configuration is checked by linearity in the
source set against oracle-computable subsets.
"""
import math

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


def check_source(bg, g, s, oracle_mod):
    got = bg.single_source(int(s))
    ref = oracle_mod.single_source(g, int(s))
    assert np.array_equal(got["d"], ref["d"]), f"d mismatch for source {s}"
    small = ref["sigma"] < TWO53
    assert np.array_equal(got["sigma"][small], ref["sigma"][small]), f"sigma mismatch, source {s}"
    assert rel_err(got["sigma"], ref["sigma"]) < 1e-12
    assert rel_err(got["delta"], ref["delta"]) < BC_TOL
    assert got["num_levels"] == ref["num_levels"]
    return got, ref


def check_bc(bg, g, sources, oracle_mod, nthreads=8):
    got = bg.compute(sources)
    ref = oracle_mod.bc(g, sources, nthreads=nthreads)
    err = rel_err(got, ref)
    assert err <= BC_TOL, f"BC max rel err {err}"
    return got, ref


STRATS = ["we", "ep", "hybrid", "sampling"]


# --------------------------------------------------------------------- C1


@pytest.mark.parametrize("strategy", STRATS)
def test_c1_exact_bc_all_sources(bcmod, oracle_mod, strategy):
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g, strategy=strategy) as bg:
        check_bc(bg, g, None, oracle_mod)
        st = bg.stats()
        assert st["sources"] == g.n
        if strategy == "we":
            assert st["ep_levels"] == 0
        if strategy == "ep":
            assert st["we_levels"] == 0


def test_c1_every_source_d_sigma_delta(bcmod, oracle_mod):
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g, strategy="we") as bg:
        for s in range(g.n):
            check_source(bg, g, s, oracle_mod)


def test_c1_stats_match_oracle_counters(bcmod, oracle_mod):
    g = graph("c1")
    src = gg.sample_sources(g, 200, seed=3)
    for strategy in ("we", "ep"):
        with bcmod.BCGraph.from_graph(g, strategy=strategy) as bg:
            bg.compute(src)
            st = bg.stats()
        refs = [oracle_mod.single_source(g, int(s)) for s in src]
        assert st["n_reached"] == sum(r["n_reached"] for r in refs)
        assert st["arcs_reached"] == sum(r["arcs_reached"] for r in refs)
        assert st["dag_arcs"] == sum(r["dag_arcs"] for r in refs)
        assert st["levels"] == sum(r["num_levels"] for r in refs)


# --------------------------------------------------------------------- C2


def test_c2_lattice_exact_bc(bcmod, oracle_mod):
    g = graph("c2")
    with bcmod.BCGraph.from_graph(g) as bg:
        check_bc(bg, g, None, oracle_mod)
        st = bg.stats()
        assert st["sampling_ep"] == 0          # median depth ~ 256+ >= 4*16 -> WE
        assert st["ep_levels"] == 0


def test_c2_lattice_sigma_beyond_2p53_bit_exact(bcmod, oracle_mod):
    """Every lattice vertex has <= 2 predecessors, so fp64 sigma is order-independent
    even at 2^505: the GPU must match the oracle bit for bit."""
    g = graph("c2")
    with bcmod.BCGraph.from_graph(g, strategy="we") as bg:
        top = 0.0
        for s in (0, 255, 65535, 128 * 256 + 77):
            got, ref = check_source(bg, g, s, oracle_mod)
            top = max(top, ref["sigma"].max())
            assert np.array_equal(got["sigma"], ref["sigma"])
        assert top > 2.0 ** 500          # corner sources: C(510, 255) ~ 2^505


def test_c2d_delaunay_subset(bcmod, oracle_mod):
    g = graph("c2d")
    src = gg.sample_sources(g, 2048, seed=5)
    with bcmod.BCGraph.from_graph(g) as bg:
        check_bc(bg, g, src, oracle_mod)
        for s in src[:8]:
            check_source(bg, g, s, oracle_mod)


# --------------------------------------------------------------------- C3


def test_c3_rgg_subset(bcmod, oracle_mod):
    g = graph("c3")
    src = gg.CONFIGS["c3"].sources(g)[:1024]
    with bcmod.BCGraph.from_graph(g) as bg:
        check_bc(bg, g, src, oracle_mod)
        st = bg.stats()
        assert st["sampling_ep"] == 0
        for s in src[:6]:
            check_source(bg, g, s, oracle_mod)


# --------------------------------------------------------------------- C4


@pytest.mark.parametrize("strategy", STRATS)
def test_c4_kron_subset(bcmod, oracle_mod, strategy):
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:600]
    with bcmod.BCGraph.from_graph(g, strategy=strategy) as bg:
        check_bc(bg, g, src, oracle_mod)
        st = bg.stats()
        if strategy == "sampling":
            assert st["sampling_ep"] == 1      # median depth ~6 < 4*18
            assert st["ep_levels"] > 0
        for s in src[:4]:
            check_source(bg, g, s, oracle_mod)


def test_c4_full_size_linearity(bcmod, oracle_mod):
    """Bench configuration (16,384 sources, default strategy): BC is linear in the
    source multiset, so GPU(S) - GPU(S minus S1) must equal oracle(S1)."""
    g = graph("c4")
    S = gg.CONFIGS["c4"].sources(g)
    rng = np.random.default_rng(11)
    pick = np.zeros(S.size, dtype=bool)
    pick[rng.choice(S.size, 48, replace=False)] = True
    with bcmod.BCGraph.from_graph(g) as bg:
        full = bg.compute(S)
        rest = bg.compute(S[~pick])
    ref = oracle_mod.bc(g, S[pick], nthreads=8)
    scale = max(1.0, float(np.abs(full).max()))
    assert float(np.abs((full - rest) - ref).max()) <= BC_TOL * scale


# ------------------------------------------------------------- selectors


def test_hybrid_modes_replay_alg4(bcmod, oracle_mod):
    from oracle import selectors as sel
    for key in ("c1", "c4"):
        g = graph(key)
        srcs = gg.sample_sources(g, 12, seed=9)
        with bcmod.BCGraph.from_graph(g, strategy="hybrid") as bg:
            for s in srcs:
                got = bg.single_source(int(s))
                ref = oracle_mod.single_source(g, int(s))
                assert got["level_modes"].tolist() == sel.hybrid_modes(ref["level_sizes"].tolist())


def test_sampling_decision_replay_alg5(bcmod, oracle_mod):
    from oracle import selectors as sel
    for key, k in (("c1", 700), ("c4", 700)):
        g = graph(key)
        src = gg.CONFIGS[key].sources(g)[:k] if key == "c4" else gg.sample_sources(g, k, seed=1)
        with bcmod.BCGraph.from_graph(g, strategy="sampling") as bg:
            bg.compute(src)
            st = bg.stats()
            depths = [oracle_mod.single_source(g, int(s))["num_levels"] - 1 for s in src[:512]]
            keys = sorted(depths)
            assert st["sampling_median"] == keys[len(keys) // 2]
            ep_run = sel.sampling_decision(depths, g.n)
            assert st["sampling_ep"] == int(ep_run)
            for s in src[512:520]:
                got = bg.single_source(int(s))
                ref = oracle_mod.single_source(g, int(s))
                assert got["level_modes"].tolist() == sel.sampling_modes(ref["level_sizes"].tolist(), ep_run)


def test_sampling_fewer_sources_than_samples(bcmod, oracle_mod):
    g = graph("c1")
    src = gg.sample_sources(g, 100, seed=2)
    with bcmod.BCGraph.from_graph(g) as bg:
        check_bc(bg, g, src, oracle_mod)
        st = bg.stats()
        assert st["ep_levels"] == 0 and st["sampling_median"] >= 0


# ------------------------------------------------------------- edge cases


def small_graphs():
    return [
        gg.star_graph(300),                     # hub of degree 299: CTA-cooperative rows
        gg.complete_graph(40),
        gg.path_graph(700),                     # 700 levels, tiny frontiers
        gg.cycle_graph(513),
        gg.csr_from_edges(6, np.array([], dtype=np.int64), np.array([], dtype=np.int64)),
        gg.csr_from_edges(9, np.array([0, 1, 4, 5]), np.array([1, 2, 5, 6])),
        gg.gnp(300, 0.02, seed=3, directed=True),
        gg.directed_path(50),
        gg.cycle_graph(40, directed=True),
        gg.rmat(11, 16, seed=8, directed=True),
        gg.lattice2d(1, 1),
    ]


@pytest.mark.parametrize("gi", range(11))
@pytest.mark.parametrize("strategy", STRATS)
def test_edge_case_graphs(bcmod, oracle_mod, gi, strategy):
    g = small_graphs()[gi]
    with bcmod.BCGraph.from_graph(g, strategy=strategy, ep_min_frontier=1, beta=1, alpha=0) as bg:
        check_bc(bg, g, None, oracle_mod)
        for s in range(min(g.n, 5)):
            check_source(bg, g, s, oracle_mod)


def test_zero_sources_duplicates_and_subsets(bcmod, oracle_mod):
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g) as bg:
        assert np.all(bg.compute(np.zeros(0, dtype=np.int32)) == 0)
        dup = np.array([3, 3, 3, 17, 900, 17], dtype=np.int32)
        check_bc(bg, g, dup, oracle_mod)
        from paper_conf_sc_mclaughlinb14_b200 import BCError
        with pytest.raises(BCError):
            bg.compute(np.array([g.n], dtype=np.int32))
        with pytest.raises(BCError):
            bg.single_source(-1)


def test_inflight_option_and_small_grids(bcmod, oracle_mod):
    g = graph("c1")
    for inflight in (1, 3, 37):
        with bcmod.BCGraph.from_graph(g, inflight=inflight) as bg:
            check_bc(bg, g, gg.sample_sources(g, 300, seed=4), oracle_mod)
            assert bg.stats()["inflight"] <= inflight


def test_backward_we_option(bcmod, oracle_mod):
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:64]
    with bcmod.BCGraph.from_graph(g, strategy="ep", backward_we=1) as bg:
        check_bc(bg, g, src, oracle_mod)


def test_determinism(bcmod):
    g = graph("c3")
    with bcmod.BCGraph.from_graph(g) as bg:
        a = bg.single_source(12345)
        b = bg.single_source(12345)
    assert np.array_equal(a["d"], b["d"]) and np.array_equal(a["sigma"], b["sigma"])


def test_compute_device_with_torch_stream(bcmod, oracle_mod):
    import torch
    g = graph("c1")
    src = gg.sample_sources(g, 333, seed=6)
    with bcmod.BCGraph.from_graph(g) as bg:
        host = bg.compute(src)
        s = torch.cuda.Stream()
        d_src = torch.from_numpy(src).cuda()
        out = torch.full((g.n,), 7.0, dtype=torch.float64, device="cuda")
        bg.compute_device(d_src, out, stream=s)
        s.synchronize()
        dev = out.cpu().numpy()
        assert rel_err(dev, host) <= 1e-12
        bg.compute_device(None, out)      # all sources, default stream
        torch.cuda.synchronize()
        assert rel_err(out.cpu().numpy(), oracle_mod.bc(g, nthreads=8)) <= BC_TOL


def test_multi_shard_sum_equals_whole(bcmod, oracle_mod):
    """Fake multi-GPU on one device: P shards computed separately and
    summed equal the whole -- the partitioning has no inter-shard dependence."""
    from paper_conf_sc_mclaughlinb14_b200 import distributed as dist
    g = graph("c4")
    S = gg.CONFIGS["c4"].sources(g)[:2000]
    with bcmod.BCGraph.from_graph(g) as bg:
        whole = bg.compute(S)
        for P in (2, 3, 8):
            parts = [bg.compute(dist.shard_sources(S, r, P, seed=4)) for r in range(P)]
            assert rel_err(np.sum(parts, axis=0), whole) <= 1e-12


@pytest.mark.parametrize("reorder", ["0", "1"])
def test_internal_reordering_is_invisible(bcmod, oracle_mod, monkeypatch, reorder):
    """The degree-ordered internal relabelling (BC_REORDER) must not change any
    output: BC, d, sigma, delta and the per-level modes are in the caller's ids."""
    monkeypatch.setenv("BC_REORDER", reorder)
    for g in (graph("c1"), gg.gnp(300, 0.02, seed=3, directed=True), gg.star_graph(500)):
        with bcmod.BCGraph.from_graph(g, strategy="sampling", ep_min_frontier=1) as bg:
            src = gg.sample_sources(g, min(200, int((g.degrees() > 0).sum())), seed=1)
            check_bc(bg, g, src, oracle_mod)
            check_bc(bg, g, None, oracle_mod)
            for s in src[:5]:
                check_source(bg, g, s, oracle_mod)


@pytest.mark.parametrize("level_store", [1, 2, 3])
@pytest.mark.parametrize("strategy", ["we", "sampling"])
def test_level_stores_agree(bcmod, oracle_mod, level_store, strategy):
    """Exact int32 d in HBM (1), 2-bit codes in shared memory (2) and 2-bit codes
    in HBM/L2 (3) are interchangeable representations of d."""
    for key, k in (("c1", None), ("c4", 300)):
        g = graph(key)
        src = None if k is None else gg.CONFIGS[key].sources(g)[:k]
        with bcmod.BCGraph.from_graph(g, strategy=strategy, level_store=level_store,
                                      ep_min_frontier=64) as bg:
            check_bc(bg, g, src, oracle_mod)
            s0 = int(src[0]) if src is not None else 7
            check_source(bg, g, s0, oracle_mod)


@pytest.mark.parametrize("key", ["c5ws", "c5k"])
def test_c5_subset_global_codes(bcmod, oracle_mod, key):
    """Largest configs (n = 2^22, level codes in HBM/L2): BC over a seeded subset of the
    config's sources and per-source d/sigma/delta against the oracle."""
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:48]
    with bcmod.BCGraph.from_graph(g) as bg:
        assert bg.options()["strategy"] == bcmod.STRATEGIES["sampling"]
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        for s in src[:2]:
            check_source(bg, g, s, oracle_mod)


@pytest.mark.parametrize("sort_frontier", [-1, 1])
def test_sorted_frontier_rebuild(bcmod, oracle_mod, sort_frontier):
    """Levels rebuilt in vertex order from the discovery bitmap (any order of S within a
    level is valid, R14) give identical d/sigma and BC within tolerance."""
    for key, k in (("c1", None), ("c3", 200), ("c4", 200)):
        g = graph(key)
        src = None if k is None else gg.CONFIGS[key].sources(g)[:k]
        with bcmod.BCGraph.from_graph(g, strategy="we", sort_frontier=sort_frontier) as bg:
            check_bc(bg, g, src, oracle_mod)
            check_source(bg, g, 5 if src is None else int(src[1]), oracle_mod)


@pytest.mark.parametrize("succ_bits", [-1, 1])
@pytest.mark.parametrize("case", [("c1", "we", 0), ("c1", "hybrid", 0), ("c2d", "we", 0),
                                  ("c3", "we", 3), ("c4", "we", 2), ("c4", "we", 3),
                                  ("c4", "ep", 0), ("c4", "sampling", 1)])
def test_successor_bitmap(bcmod, oracle_mod, succ_bits, case):
    """The successor bitmap (one bit per arc set in the forward scan, read by the backward
    sweep) only skips non-successor arcs: d/sigma/delta and BC are unchanged."""
    key, strategy, lstore = case
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:150]
    with bcmod.BCGraph.from_graph(g, strategy=strategy, succ_bits=succ_bits,
                                  level_store=lstore) as bg:
        check_bc(bg, g, src, oracle_mod)
        check_source(bg, g, int(src[2]), oracle_mod)
        check_source(bg, g, int(src[2]), oracle_mod)  # bitmap cleared between sources


def test_trace_source_levels(bcmod, oracle_mod):
    """N2 per-level trace: frontier sizes equal the oracle's level sizes exactly."""
    for key in ("c1", "c3", "c4"):
        g = graph(key)
        s = int(gg.CONFIGS[key].sources(g)[3])
        with bcmod.BCGraph.from_graph(g, strategy="we") as bg:
            tr = bg.trace_source(s)
        ref = oracle_mod.single_source(g, s)
        assert tr["num_levels"] == ref["num_levels"]
        assert np.array_equal(tr["level_sizes"], ref["level_sizes"])
        assert np.all(tr["fwd_cycles"] > 0)
        assert np.all(tr["bwd_cycles"][1:-1] > 0) and tr["bwd_cycles"][0] == 0


@pytest.mark.parametrize("flags", [(1, 0), (0, 1), (1, 1)])
def test_extrapolate_and_normalize(bcmod, oracle_mod, flags):
    """N3 post-processing: n/k estimator scaling and the (n-1)(n-2) normalisation."""
    extrapolate, normalize = flags
    g = graph("c1")
    src = gg.sample_sources(g, 100, seed=8)
    ref = oracle_mod.bc(g, src, nthreads=8)
    if extrapolate:
        ref = ref * g.n / src.size
    if normalize:
        ref = ref / ((g.n - 1) * (g.n - 2))
    with bcmod.BCGraph.from_graph(g, extrapolate=extrapolate, normalize=normalize) as bg:
        got = bg.compute(src)
    assert np.max(np.abs(got - ref) / np.maximum(np.abs(ref), 1e-300)) < 1e-9


@pytest.mark.parametrize("seq,warp", [(4, 8), (8, 200), (32, 4096), (128, 16384), (1024, 1024)])
def test_row_split_knobs(bcmod, oracle_mod, seq, warp):
    """Rows summed by one thread (deg <= seq), one warp (<= warp) or the whole CTA:
    every split gives identical d/sigma (integers < 2^53) and BC within tolerance."""
    for key, k in (("c1", None), ("c4", 120)):
        g = graph(key)
        src = None if k is None else gg.CONFIGS[key].sources(g)[:k]
        with bcmod.BCGraph.from_graph(g, strategy="we", seq_max_deg=seq, warp_max_deg=warp) as bg:
            check_bc(bg, g, src, oracle_mod)
            hub = int(np.argmax(g.degrees()))
            check_source(bg, g, hub, oracle_mod)
            check_source(bg, g, 3 if src is None else int(src[0]), oracle_mod)


@pytest.mark.parametrize("strategy", STRATS)
def test_fig1_consistent_golden(bcmod, oracle_mod, strategy):
    """The CUDA path on the hand-derived Figure 1 fixture (tests/golden/)."""
    import golden_io
    g, want = golden_io.load("fig1_consistent.txt")
    with bcmod.BCGraph.from_graph(g, strategy=strategy) as bg:
        for s in range(g.n):
            check_source(bg, g, s, oracle_mod)
        assert rel_err(bg.compute(None), want) < 1e-12


def test_compute_device_empty_source_tensor(bcmod):
    """An empty CUDA tensor has data_ptr() == 0; it must mean "no sources" (BC = 0), not
    the C ABI's NULL = "all vertices" (an empty multi-GPU shard)."""
    import torch
    g = graph("c1")
    with bcmod.BCGraph.from_graph(g) as bg:
        out = torch.full((g.n,), 3.0, dtype=torch.float64, device="cuda")
        bg.compute_device(torch.zeros(0, dtype=torch.int32, device="cuda"), out)
        torch.cuda.synchronize()
        assert float(out.abs().max()) == 0.0
        assert bg.stats()["sources"] == 0


def test_seq_max_deg_shrink_reallocates_bigq(bcmod, oracle_mod):
    """lowering the effective row-split threshold (seq_max_deg) must grow the
    hub-row queue (bigq); c4's hubs then all go to the CTA-cooperative phase."""
    g = graph("c4")
    src = gg.CONFIGS["c4"].sources(g)[:40]
    with bcmod.BCGraph.from_graph(g, strategy="we", seq_max_deg=20000, inflight=7) as bg:
        bg.set_options(seq_max_deg=0)   # effective threshold 20000 -> 8192: bigq must grow
        check_bc(bg, g, src, oracle_mod)
        bg.set_options(seq_max_deg=4, warp_max_deg=8)
        check_bc(bg, g, src, oracle_mod)


@pytest.mark.parametrize("key,strategy,expect_handover", [
    ("c3", "hybrid", False),     # Alg. 4 never picks EP on RGG (frontier changes < alpha)
    ("c2", "sampling", False),   # Alg. 5 decides WE on the lattice (median depth >= 64)
    ("c4", "hybrid", True),      # Alg. 4 picks EP for the Kronecker middle levels
    ("c4", "sampling", True),    # Alg. 5 decides EP; guard 512 admits EP levels
])
def test_optimistic_we_with_handover(bcmod, oracle_mod, key, strategy, expect_handover):
    """Alg. 4 / Alg. 5 with the paper's parameters run on the fast work-efficient kernel;
    a source whose selector picks an EP level is handed over (re-run from scratch) to the
    EP-capable kernel.  BC is the oracle's either way, every source is counted once, and the
    per-level modes of a handed-over source match the selector replay."""
    from oracle import selectors as sel
    g = graph(key)
    src = gg.CONFIGS[key].sources(g)[:900] if gg.CONFIGS[key].k else gg.sample_sources(g, 900, seed=12)
    with bcmod.BCGraph.from_graph(g, strategy=strategy) as bg:
        check_bc(bg, g, src, oracle_mod, nthreads=16)
        st = bg.stats()
        assert st["sources"] == src.size
        if expect_handover:
            assert st["handovers"] > 0 and st["ep_levels"] > 0
        else:
            assert st["handovers"] == 0 and st["ep_levels"] == 0
        if strategy == "hybrid":
            for s in src[:3]:
                ref = oracle_mod.single_source(g, int(s))
                assert bg.single_source(int(s))["level_modes"].tolist() == sel.hybrid_modes(ref["level_sizes"].tolist())


@pytest.mark.parametrize("key,strategy,k,inflight,extra", [
    ("c1", "sampling", 700, 0, {}),                      # paper parameters: some sources hand over
    ("c1", "hybrid", 300, 1, {"alpha": 0, "beta": 16}),  # one CTA; EP from the first big change
    ("c4", "hybrid", 120, 5, {}),
])
def test_handover_counters_and_duplicates(bcmod, oracle_mod, key, strategy, k, inflight, extra):
    """A handed-over source is counted once: its partial forward on the WE-only kernel is
    rolled back (levels, distance sum, arcs, DAG arcs) and recomputed by the EP-capable
    kernel.  The byte-model counters and the level count then equal the oracle's, and BC
    is the oracle's -- also with duplicate sources and a single CTA in flight."""
    g = graph(key)
    src = gg.sample_sources(g, k, seed=21) if key == "c1" else gg.CONFIGS[key].sources(g)[:k]
    src = np.concatenate([src, src[:7]])      # duplicates count with multiplicity (R15)
    opts = dict(strategy=strategy, inflight=inflight, **extra)
    with bcmod.BCGraph.from_graph(g, **opts) as bg:
        check_bc(bg, g, src, oracle_mod)
        st = bg.stats()
    assert st["handovers"] > 0
    refs = [oracle_mod.single_source(g, int(s)) for s in src]
    assert st["sources"] == src.size
    assert st["n_reached"] == sum(r["n_reached"] for r in refs)
    assert st["arcs_reached"] == sum(r["arcs_reached"] for r in refs)
    assert st["dag_arcs"] == sum(r["dag_arcs"] for r in refs)
    assert st["levels"] == sum(r["num_levels"] for r in refs)
    assert st["dist_sum"] == sum(int(r["d"][r["d"] >= 0].sum()) for r in refs)
