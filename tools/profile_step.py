#!/usr/bin/env python
"""One bc_compute_device step of a config, for ncu captures (no timing printed).

    ncu --set full --clock-control none --import-source on -k regex:bc_kernel \
        -c 2 -o gpurun_out/prof python tools/profile_step.py --config c4
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--strategy", default="sampling")
    ap.add_argument("--sources", type=int, default=0, help="0 = the config's source set")
    ap.add_argument("--repeat", type=int, default=1)
    ap.add_argument("--opt", action="append", default=[], help="option=value")
    ap.add_argument("--stats-out", default=None, help="write the step's stats + byte model as JSON")
    a = ap.parse_args()
    import torch
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    cfg = gg.CONFIGS[a.config]
    g = cfg.graph()
    src = cfg.sources(g)
    if a.sources:
        src = src[: a.sources]
    opts = {k: int(v) for k, v in (o.split("=") for o in a.opt)}
    bg = bcm.BCGraph.from_graph(g, strategy=a.strategy, **opts)
    d_src = torch.from_numpy(src).cuda()
    out = torch.empty(g.n, dtype=torch.float64, device="cuda")
    for _ in range(a.repeat):
        bg.compute_device(d_src, out)
    torch.cuda.synchronize()
    st = bg.stats()
    print({k: st[k] for k in ("sources", "levels", "ep_levels", "kernel_ms", "n_reached",
                              "arcs_reached", "dag_arcs", "inflight")}, file=sys.stderr)
    if a.stats_out:
        import json
        # SURVEY 8(d) byte model, per launch-step (all bc_kernel launches of the step)
        alg = (20.0 * g.n * st["sources"] + 16.0 * st["arcs_reached"] + 24.0 * st["dag_arcs"]
               + 64.0 * st["n_reached"])
        json.dump({"config": a.config, "strategy": a.strategy, "sources": int(src.size),
                   "stats": st, "alg_bytes_per_step": alg, "launches": st["bc_kernel_launches"]},
                  open(a.stats_out, "w"), indent=1)
    bg.close()


if __name__ == "__main__":
    main()
