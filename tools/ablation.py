#!/usr/bin/env python
"""Strategy ablation on B200 (the paper's Fig. 4 analog):
pure work-efficient (WE), pure edge-parallel (EP), hybrid (Alg. 4) and sampling
(Alg. 5) with the paper's parameters on each config, then one-at-a-time sweeps of the
paper's constants around their published values: alpha, beta (Alg. 4), gamma
(P:299), n_samps and the EP guard.

    python tools/ablation.py --configs c1,c2,c2d,c3,c4,c5ws,c5k --out profiles/r02/ablation.json
    python tools/ablation.py --table profiles/r02/ablation.json > profiles/r02/ablation.md

Kernel time = bc_stats.kernel_ms (CUDA events around the traversal launches) of the second
of two identical compute calls (the first warms up); GTEPS = m x sources / time.
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

SOURCES = {"c1": None, "c2": 8192, "c2d": 8192, "c3": 2048, "c4": 4096, "c5ws": 1024, "c5k": 1024}
PAPER = {"alpha": 768, "beta": 512, "gamma": 4.0, "n_samps": 512, "ep_min_frontier": 512}
SWEEPS = {
    "alpha": ("hybrid", [128, 768, 4096, 32768]),
    "beta": ("hybrid", [64, 512, 4096, 32768]),
    "gamma": ("sampling", [1.0, 2.0, 4.0, 8.0]),
    "n_samps": ("sampling", [64, 256, 512, 2048]),
    "ep_min_frontier": ("sampling", [512, 8192, 65536, 2147483647]),
}


def table(path):
    d = json.load(open(path))
    rows = d["rows"]
    cfgs = list(dict.fromkeys(r["config"] for r in rows))
    base = [r for r in rows if r["sweep"] == "strategy"]
    print(f"# N1 strategy ablation (B200, kernel GTEPS; {d['when']}, HEAD {d.get('head', '?')})\n")
    print("Paper parameters: alpha 768, beta 512, gamma 4, n_samps 512, EP guard 512.\n")
    print("| config | sources | WE | EP | hybrid (Alg. 4) | sampling (Alg. 5) | sampling, B200 guard |")
    print("|---|---|---|---|---|---|---|")
    for c in cfgs:
        rs = {r["label"]: r for r in base if r["config"] == c}
        def v(lbl):
            r = rs.get(lbl)
            if not r:
                return "-"
            extra = f" ({r['ep_levels']} EP lv, {r['handovers']} h/o)" if r["ep_levels"] or r["handovers"] else ""
            return f"{r['gteps']:.1f}{extra}"
        k = next(iter(rs.values()))["sources"]
        print(f"| {c} | {k} | {v('we')} | {v('ep')} | {v('hybrid')} | {v('sampling')} | {v('sampling_b200')} |")
    for name, (strat, vals) in SWEEPS.items():
        sw = [r for r in rows if r["sweep"] == name]
        if not sw:
            continue
        print(f"\n## {name} sweep ({strat}; paper value {PAPER[name]})\n")
        print("| config | " + " | ".join(str(x) for x in vals) + " |")
        print("|---|" + "---|" * len(vals))
        for c in cfgs:
            rs = {r["value"]: r for r in sw if r["config"] == c}
            if rs:
                print(f"| {c} | " + " | ".join(f"{rs[x]['gteps']:.1f}" if x in rs else "-" for x in vals) + " |")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c1,c2,c2d,c3,c4")
    ap.add_argument("--sweep-configs", default="c2,c3,c4,c5ws,c5k")
    ap.add_argument("--out", default=None)
    ap.add_argument("--table", default=None, help="print the markdown tables of a saved JSON")
    a = ap.parse_args()
    if a.table:
        table(a.table)
        return
    import torch
    import paper_conf_sc_mclaughlinb14_b200 as bcm
    from paper_conf_sc_mclaughlinb14_b200 import graphgen as gg
    rows = []
    head = os.environ.get("BC_HEAD") or os.popen("git rev-parse --short HEAD 2>/dev/null").read().strip() or None

    def run(g, key, src, d_src, out, strategy, sweep, label, value, opts):
        bg = bcm.BCGraph.from_graph(g, strategy=strategy, **opts)
        for _ in range(2):
            bg.compute_device(d_src, out)
            torch.cuda.synchronize()
        st = bg.stats()
        bg.close()
        ms = st["kernel_ms"]
        row = {"config": key, "graph": g.name, "n": g.n, "m": g.m, "sources": int(src.size),
               "strategy": strategy, "sweep": sweep, "label": label, "value": value, "opts": opts,
               "kernel_ms": round(ms, 3), "gteps": round(g.m * src.size / (ms / 1e3) / 1e9, 3),
               "ep_levels": st["ep_levels"], "we_levels": st["we_levels"], "handovers": st["handovers"],
               "engines": st["engines"], "sampling_ep": st["sampling_ep"],
               "sampling_median": st["sampling_median"],
               "arcs_scanned_per_teps_edge": round(st["arcs_scanned"] / (g.m * src.size), 3)}
        print(json.dumps(row), flush=True)
        rows.append(row)

    keys = list(dict.fromkeys(a.configs.split(",") + a.sweep_configs.split(",")))
    for key in keys:
        cfg = gg.CONFIGS[key]
        g = cfg.graph()
        src = cfg.sources(g)
        k = SOURCES.get(key)
        if k:
            src = src[:k]
        d_src = torch.from_numpy(src).cuda()
        out = torch.empty(g.n, dtype=torch.float64, device="cuda")
        if key in a.configs.split(","):
            for label, strat, opts in (("we", "we", {}), ("ep", "ep", {}), ("hybrid", "hybrid", {}),
                                       ("sampling", "sampling", {}),
                                       ("sampling_b200", "sampling", {"ep_min_frontier": 2147483647})):
                run(g, key, src, d_src, out, strat, "strategy", label, None, opts)
        if key in a.sweep_configs.split(","):
            for name, (strat, vals) in SWEEPS.items():
                for v in vals:
                    run(g, key, src, d_src, out, strat, name, f"{name}={v}", v, {name: v})
        del g
    if a.out:
        json.dump({"when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()), "head": head, "rows": rows},
                  open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
