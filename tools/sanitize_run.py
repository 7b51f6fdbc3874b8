#!/usr/bin/env python
"""One small BC computation per engine, for compute-sanitizer runs (memcheck, racecheck,
synccheck):

    compute-sanitizer --tool racecheck python tools/sanitize_run.py --graph c1 --engine group

Graphs: c1 (R-MAT s10, all 1,024 sources) or lat64 (64 x 64 lattice, 4,096 vertices,
126 levels, sources = every 8th vertex).  Engines: per_source (strategies WE, EP, hybrid,
sampling), group (WE), batched (WE).  Each result is compared with the oracle (1e-9)."""
import argparse
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", default="c1", choices=["c1", "lat64"])
    ap.add_argument("--engine", default="per_source", choices=["per_source", "group", "batched"])
    ap.add_argument("--stride", type=int, default=8, help="lat64: sources = every stride-th vertex")
    a = ap.parse_args()
    import oracle
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    if a.graph == "c1":
        g = gg.CONFIGS["c1"].graph()
        src = None
    else:
        g = gg.lattice2d(64, 64)
        src = np.arange(0, g.n, a.stride, dtype=np.int32)
    strategies = ["we", "ep", "hybrid", "sampling"] if a.engine == "per_source" else ["we"]
    ref = oracle.bc(g, src, nthreads=8)
    worst = 0.0
    for strat in strategies:
        extra = dict(ep_min_frontier=16, beta=16, alpha=0) if strat != "we" else {}
        with bcm.BCGraph.from_graph(g, strategy=strat, engine=a.engine, **extra) as bg:
            got = bg.compute(src)
            one = bg.single_source(3) if a.engine != "batched" else None
        err = float(np.max(np.abs(got - ref) / np.maximum(np.abs(ref), 1.0)))
        worst = max(worst, err)
        print(f"{a.graph} {a.engine} {strat}: max rel err {err:.2e}", flush=True)
        if one is not None:
            r1 = oracle.single_source(g, 3)
            assert np.array_equal(one["d"], r1["d"])
    assert worst <= 1e-9, worst
    print("SANITIZE_RUN_OK")


if __name__ == "__main__":
    main()
