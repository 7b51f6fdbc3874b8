#!/usr/bin/env python
"""A/B timing of libbc builds (select one with BC_LIBBC=path/libbc.so): kernel ms of one
bc_compute_device step per config (median of --reps after one warm-up), plus the BC vector
saved for a cross-build comparison (tools/ab_time.py --compare a.npy b.npy).

    BC_LIBBC=build/base/libbc.so python tools/ab_time.py --tag base --spec c4:16384 --spec c3:8192
"""
import argparse
import hashlib
import json
import os
import statistics
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="default")
    ap.add_argument("--spec", action="append", default=[], help="config:sources[:opt=v,...]")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/ab")
    ap.add_argument("--compare", nargs=2, default=None)
    ap.add_argument("--save-max-n", type=int, default=1 << 19, help="save BC vectors only for n <= this")
    a = ap.parse_args()
    if a.compare:
        x, y = np.load(a.compare[0]), np.load(a.compare[1])
        print(json.dumps({"compare": a.compare, "max_rel": float(np.max(np.abs(x - y) / np.maximum(np.abs(y), 1.0)))}))
        return
    import torch
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    os.makedirs(a.out, exist_ok=True)
    graphs = {}
    for spec in a.spec:
        parts = spec.split(":")
        key, k = parts[0], int(parts[1])
        opts = {"strategy": "sampling", "ep_min_frontier": 2147483647}
        if len(parts) > 2 and parts[2]:
            for kv in parts[2].split(","):
                kk, vv = kv.split("=")
                opts[kk] = int(vv) if vv.lstrip("-").isdigit() else vv
        if key not in graphs:
            graphs[key] = gg.CONFIGS[key].graph()
        g = graphs[key]
        src = gg.CONFIGS[key].sources(g)
        if k:
            src = src[:k]
        with bcm.BCGraph.from_graph(g, **opts) as bg:
            d_src = torch.from_numpy(src).cuda()
            out = torch.empty(g.n, dtype=torch.float64, device="cuda")
            bg.compute_device(d_src, out)
            torch.cuda.synchronize()
            ms = []
            for _ in range(a.reps):
                bg.compute_device(d_src, out)
                torch.cuda.synchronize()
                ms.append(bg.stats()["kernel_ms"])
            st = bg.stats()
        name = f"{a.tag}_{key}_{k}_{hashlib.md5(str(sorted(opts.items())).encode()).hexdigest()[:8]}"
        if g.n <= a.save_max_n:
            np.save(os.path.join(a.out, name + ".npy"), out.cpu().numpy())
        gteps = g.m * src.size / (statistics.median(ms) / 1e3) / 1e9
        print(json.dumps({"tag": a.tag, "config": key, "sources": int(src.size), "opts": opts,
                          "kernel_ms": statistics.median(ms), "all_ms": ms, "gteps": gteps,
                          "engines": st["engines"], "phase_cycles": st["phase_cycles"], "levels": st["levels"],
                          "arcs_scanned": st["arcs_scanned"], "group_wait_cycles": st.get("group_wait_cycles", 0),
                          "group_mode": st.get("group_mode", -1), "inflight": st["inflight"],
                          "file": name}), flush=True)


if __name__ == "__main__":
    main()
