#!/usr/bin/env python
"""Summarise an ncu report: headline throughput metrics, DRAM/L2 bytes, stall
reasons and the hottest SASS instructions (with source lines when available).

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--top 25] [--out profiles/x.txt]
"""
import argparse
import csv
import io
import subprocess
import sys


def ncu_csv(rep, *args):
    out = subprocess.run(["ncu", "-i", rep, "--csv", *args], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


HEAD = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum", "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "smsp__inst_executed.sum"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--top", type=int, default=25)
    ap.add_argument("--out")
    a = ap.parse_args()
    lines = []
    raw = ncu_csv(a.rep, "--page", "raw")
    if len(raw) < 3:
        print("no data", file=sys.stderr)
        return 1
    h, u, v = raw[0], raw[1], raw[2]
    d = {n: (val, un) for n, un, val in zip(h, u, v)}
    lines.append(f"report: {a.rep}")
    lines.append(f"kernel: {d.get('Kernel Name', ('?', ''))[0]}")
    for k in HEAD:
        if k in d:
            lines.append(f"  {k:70s} {d[k][0]:>20s} {d[k][1]}")
    stalls = []
    for n, (val, un) in d.items():
        if n.startswith("smsp__pcsamp_warps_issue_stalled_") and not n.endswith("_not_issued"):
            try:
                stalls.append((float(val), n.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            except ValueError:
                pass
    tot = sum(s for s, _ in stalls) or 1.0
    lines.append("stall reasons (share of PC samples):")
    for s, n in sorted(stalls, reverse=True)[:10]:
        lines.append(f"  {n:40s} {100 * s / tot:6.2f}%")
    src = ncu_csv(a.rep, "--page", "source", "--print-source", "sass")
    if len(src) > 2:
        hh = src[1]
        idx = {n: i for i, n in enumerate(hh)}
        rows = src[2:]
        key = "Warp Stall Sampling (All Samples)"
        tot = sum(float(r[idx[key]] or 0) for r in rows) or 1.0
        lines.append(f"top {a.top} SASS instructions by stall samples:")
        for r in sorted(rows, key=lambda r: -float(r[idx[key]] or 0))[: a.top]:
            lines.append(f"  {100 * float(r[idx[key]]) / tot:6.2f}%  {r[idx['Source']][:60]:60s} "
                         f"exec={r[idx['Instructions Executed']]}")
    text = "\n".join(lines)
    print(text)
    if a.out:
        open(a.out, "w").write(text + "\n")
    return 0


if __name__ == "__main__":
    sys.exit(main())
