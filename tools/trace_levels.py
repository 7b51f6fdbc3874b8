#!/usr/bin/env python
"""Per-level frontier sizes and forward/backward SM cycles of a few sources (N2 trace,
bc_trace_source), to see where a config's time goes (small latency-bound levels vs large
throughput-bound ones).  Uses the engine the config's bench options select.

    python tools/trace_levels.py --config c5ws --n 3
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5ws")
    ap.add_argument("--n", type=int, default=3)
    ap.add_argument("--opt", action="append", default=[])
    a = ap.parse_args()
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    cfg = gg.CONFIGS[a.config]
    g = cfg.graph()
    src = cfg.sources(g)[: a.n]
    opts = {"strategy": "sampling", "ep_min_frontier": 2147483647}
    for o in a.opt:
        k, v = o.split("=")
        opts[k] = int(v)
    deg = g.degrees()
    import numpy as np
    with bcm.BCGraph.from_graph(g, **opts) as bg:
        for s in src:
            tr = bg.trace_source(int(s))
            one = bg.single_source(int(s))
            d = one["d"]
            tot_f = tr["fwd_cycles"].sum()
            tot_b = tr["bwd_cycles"].sum()
            print(f"source {s}: levels {tr['num_levels']}, fwd {tot_f/1e6:.2f} Mcyc, bwd {tot_b/1e6:.2f} Mcyc")
            for L in range(tr["num_levels"]):
                arcs = int(deg[d == L].sum())
                print(f"  L={L:3d} size={tr['level_sizes'][L]:9d} arcs={arcs:10d} fwd={tr['fwd_cycles'][L]/1e3:9.1f}k "
                      f"bwd={tr['bwd_cycles'][L]/1e3:9.1f}k  fwd cyc/arc={tr['fwd_cycles'][L]/max(arcs,1):7.3f}")


if __name__ == "__main__":
    main()
