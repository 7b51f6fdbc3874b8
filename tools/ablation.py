#!/usr/bin/env python
"""Strategy ablation on B200 (the paper's Fig. 4 analog):
pure work-efficient (WE), pure edge-parallel (EP), hybrid (Alg. 4) and sampling
(Alg. 5) with the paper's parameters, on each config, plus an EP-guard sweep.

    python tools/ablation.py --configs c1,c2,c3,c4,c5ws,c5k --out profiles/r01/ablation.json
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

SOURCES = {"c1": None, "c2": 8192, "c2d": 8192, "c3": 2048, "c4": 4096, "c5ws": 1024, "c5k": 768}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c1,c2,c3,c4")
    ap.add_argument("--guards", default="512,8192,65536,1000000000")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    rows = []
    for key in a.configs.split(","):
        cfg = gg.CONFIGS[key]
        g = cfg.graph()
        src = cfg.sources(g)
        k = SOURCES.get(key)
        if k:
            src = src[:k]
        d_src = torch.from_numpy(src).cuda()
        out = torch.empty(g.n, dtype=torch.float64, device="cuda")
        runs = [("we", {}), ("ep", {}), ("hybrid", {}), ("sampling", {})]
        runs += [("sampling", {"ep_min_frontier": int(x)}) for x in a.guards.split(",") if int(x) != 512]
        for strat, extra in runs:
            bg = bcm.BCGraph.from_graph(g, strategy=strat, **extra)
            bg.compute_device(d_src, out)
            torch.cuda.synchronize()
            bg.compute_device(d_src, out)
            torch.cuda.synchronize()
            st = bg.stats()
            ms = st["kernel_ms"]
            row = {"config": key, "graph": g.name, "n": g.n, "m": g.m, "sources": int(src.size),
                   "strategy": strat, "opts": extra, "kernel_ms": round(ms, 3),
                   "gteps": round(g.m * src.size / (ms / 1e3) / 1e9, 3),
                   "ep_levels": st["ep_levels"], "we_levels": st["we_levels"],
                   "sampling_ep": st["sampling_ep"], "sampling_median": st["sampling_median"],
                   "arcs_scanned_per_teps_edge": round(st["arcs_scanned"] / (g.m * src.size), 3)}
            print(json.dumps(row), flush=True)
            rows.append(row)
            bg.close()
    if a.out:
        json.dump({"when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()), "rows": rows},
                  open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
