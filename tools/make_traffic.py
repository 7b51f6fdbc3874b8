#!/usr/bin/env python
"""Combine an ncu capture of ALL bc_kernel launches of one step (DRAM bytes) with
the step's algorithmic byte model (tools/profile_step.py --stats-out) into
profiles/traffic.json: {config: {"dram_bytes_per_alg_byte": r, ...}}, which bench.py
uses to report roofline.traffic per step.

    python tools/make_traffic.py gpurun_out/prof.ncu-rep gpurun_out/stats.json [--out profiles/traffic.json]
"""
import argparse
import csv
import io
import json
import os
import subprocess


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("stats")
    ap.add_argument("--out", default="profiles/traffic.json")
    a = ap.parse_args()
    out = subprocess.run(["ncu", "-i", a.rep, "--csv", "--page", "raw", "--metrics",
                          "dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,gpu__time_duration.sum"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    dram = 0.0
    lts = 0.0
    dur = 0.0
    kernels = 0
    for r in rows[2:]:
        d = dict(zip(h, r))
        if not any(k in d.get("Kernel Name", "") for k in ("bc_kernel", "group_kernel", "batch_kernel")):
            continue
        kernels += 1
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            dram += float(d[k]) * scale.get(rows[1][h.index(k)], 1)
        if "lts__t_bytes.sum" in d and d["lts__t_bytes.sum"] not in ("", "n/a"):
            lts += float(d["lts__t_bytes.sum"]) * scale.get(rows[1][h.index("lts__t_bytes.sum")], 1)
        tunit = rows[1][h.index("gpu__time_duration.sum")]
        dur += float(d["gpu__time_duration.sum"]) * {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3, "s": 1e3}.get(tunit, 1.0)
    st = json.load(open(a.stats))
    res = json.load(open(a.out)) if os.path.exists(a.out) else {}
    res[st["config"]] = {"strategy": st["strategy"], "sources": st["sources"],
                         "bc_kernel_launches_captured": kernels, "dram_bytes": dram,
                         "alg_bytes": st["alg_bytes_per_step"],
                         "dram_bytes_per_alg_byte": dram / st["alg_bytes_per_step"],
                         "lts_bytes": lts, "lts_bytes_per_alg_byte": (lts / st["alg_bytes_per_step"]) if lts else None,
                         "kernel_ms_under_ncu": dur,
                         "source": os.path.basename(a.rep)}
    json.dump(res, open(a.out, "w"), indent=1)
    print(json.dumps(res[st["config"]]))


if __name__ == "__main__":
    main()
