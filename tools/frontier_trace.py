#!/usr/bin/env python
"""N2: the paper's Table I / Fig. 3 study on the synthetic
analogs, on B200.  For three roots per graph, the per-level forward time (SM cycles of
the one CTA that owns the source, work-efficient expansion, bc_trace_source) is
correlated with the vertex-frontier size (rho_v,t) and the edge-frontier size
(rho_e,t = sum of degrees of the level's vertices); the frontier as % of n per level
is the Fig. 3 curve.

    python tools/frontier_trace.py --out profiles/r01/table1_analog.json
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c2,c2d,c3,c4,c5ws")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    rows = []
    for key in a.configs.split(","):
        g = gg.CONFIGS[key].graph()
        deg = g.degrees()
        nz = np.nonzero(deg > 0)[0]
        roots = [int(nz[i % nz.size]) for i in (0, 2121, 6004)]  # Table I's root ids, mod #non-isolated
        with bcm.BCGraph.from_graph(g, strategy="we") as bg:
            for r in roots:
                bg.trace_source(r)  # warm
                tr = bg.trace_source(r)
                one = bg.single_source(r)
                d = one["d"]
                L = tr["num_levels"]
                efront = np.bincount(d[d >= 0], weights=deg[d >= 0], minlength=L)[:L]
                t = tr["fwd_cycles"].astype(np.float64)
                v = tr["level_sizes"].astype(np.float64)
                rv = float(np.corrcoef(v, t)[0, 1]) if L > 2 else float("nan")
                re = float(np.corrcoef(efront, t)[0, 1]) if L > 2 else float("nan")
                row = {"config": key, "graph": g.name, "root": r, "levels": L,
                       "rho_v_t": round(rv, 3), "rho_e_t": round(re, 3),
                       "frontier_pct_of_n": [round(100.0 * x / g.n, 4) for x in v.tolist()],
                       "fwd_cycles": t.astype(int).tolist()}
                print(json.dumps({k: row[k] for k in ("config", "root", "levels", "rho_v_t", "rho_e_t")}),
                      flush=True)
                rows.append(row)
    if a.out:
        json.dump({"paper_table1": "P:231-249 (rgg, delaunay, kron, luxembourg, smallworld on Kepler)",
                   "rows": rows}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
