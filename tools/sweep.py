#!/usr/bin/env python
"""Option sweep for tuning: kernel time of one bc_compute_device step per setting.

    python tools/sweep.py --config c4 --sources 4096 --set strategy=we \
        --grid block_threads=256,512 --grid seq_max_deg=8,32
"""
import argparse
import itertools
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def parse_val(v):
    try:
        return int(v)
    except ValueError:
        return v


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--sources", type=int, default=0)
    ap.add_argument("--set", action="append", default=[])
    ap.add_argument("--grid", action="append", default=[])
    ap.add_argument("--reps", type=int, default=2)
    a = ap.parse_args()
    import torch
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    cfg = gg.CONFIGS[a.config]
    g = cfg.graph()
    src = cfg.sources(g)
    if a.sources:
        src = src[: a.sources]
    base = {k: parse_val(v) for k, v in (s.split("=") for s in a.set)}
    keys, vals = [], []
    for gr in a.grid:
        k, v = gr.split("=")
        keys.append(k)
        vals.append([parse_val(x) for x in v.split(",")])
    d_src = torch.from_numpy(src).cuda()
    out = torch.empty(g.n, dtype=torch.float64, device="cuda")
    ref = None
    for combo in itertools.product(*vals) if vals else [()]:
        opts = dict(base)
        opts.update(dict(zip(keys, combo)))
        bg = bcm.BCGraph.from_graph(g, **opts)
        bg.compute_device(d_src, out)
        torch.cuda.synchronize()
        best = 1e30
        for _ in range(a.reps):
            bg.compute_device(d_src, out)
            torch.cuda.synchronize()
            best = min(best, bg.stats()["kernel_ms"])
        res = out.cpu().numpy()
        if ref is None:
            ref = res
        err = float(abs(res - ref).max() / max(1.0, abs(ref).max()))
        st = bg.stats()
        gteps = g.m * src.size / (best / 1e3) / 1e9
        print(json.dumps({"config": a.config, "opts": opts, "kernel_ms": round(best, 2),
                          "gteps": round(gteps, 2), "inflight": st["inflight"],
                          "ep_levels": st["ep_levels"], "rel_diff_vs_first": err,
                          "phase_share": [round(x / max(1, sum(st["phase_cycles"])), 3)
                                          for x in st["phase_cycles"]]}), flush=True)
        bg.close()


if __name__ == "__main__":
    main()
