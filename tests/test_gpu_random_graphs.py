"""Randomised parity sweep of the late-round-2 paths on many small seeded graphs (the
compute-sanitizer is closed on this GPU pool, so races / bounds errors in the new code are
hunted by breadth instead): the per-source fast path with the backward pushed on every
level that qualifies (BC_BPUSH=1, bc_fast.cuh push_level) and the group engine's thin-row
passes (BC_GROUP_MODE=2, bc_thin.cuh), against the CPU oracle at 1e-9.
Graph kinds: R-MAT (skewed, relabelled), G(n,p) (several components), Watts-Strogatz
(ring order, no hubs), random geometric (high diameter), Delaunay-like, stars with a row
longer than the thin-row limit, and their disjoint unions."""
import numpy as np
import pytest

from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg

from test_gpu_parity import BC_TOL, bcmod, rel_err  # noqa: F401

pytestmark = pytest.mark.gpu


def graphs():
    out = []
    for seed in range(4):
        out.append(gg.rmat(9 + seed % 2, 8, seed=200 + seed))
        out.append(gg.gnp(400 + 50 * seed, 0.01, seed=300 + seed))
        out.append(gg.watts_strogatz(1500 + 100 * seed, 6 + 2 * seed, 0.1 + 0.1 * seed, seed=400 + seed))
        out.append(gg.rgg(1200 + 100 * seed, seed=500 + seed))
        out.append(gg.delaunay(900 + 100 * seed, seed=600 + seed))
    out.append(gg.star_graph(100))
    return out


@pytest.mark.parametrize("path", ["push", "thin"])
def test_random_graphs(bcmod, oracle_mod, monkeypatch, path):
    if path == "push":
        monkeypatch.setenv("BC_BPUSH", "1")
        opts = dict(strategy="we")
    else:
        monkeypatch.setenv("BC_GROUP_MODE", "2")
        opts = dict(strategy="we", engine="group", group_ctas=5)
    rng = np.random.default_rng(7)
    for i, g in enumerate(graphs()):
        src = None if g.n <= 600 else np.sort(rng.choice(g.n, 96, replace=False)).astype(np.int32)
        with bcmod.BCGraph.from_graph(g, **opts) as bg:
            got = bg.compute(src)
            st = bg.stats()
        ref = oracle_mod.bc(g, src, nthreads=16)
        err = rel_err(got, ref)
        assert err <= BC_TOL, f"graph {i} ({g.name}, n={g.n}): BC max rel err {err}"
        if path == "thin":
            assert st["group_mode"] == 2
