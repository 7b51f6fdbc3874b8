#!/usr/bin/env python
"""Per-CUDA-source-line instruction counts and stall samples from an ncu report
(ncu -i REP --page source --csv --print-source cuda,sass), sorted by warp instructions.

    python tools/ncu_lines2.py gpurun_out/full_c4_main.ncu-rep [--top 40]
"""
import argparse
import csv
import io
import subprocess


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--top", type=int, default=40)
    ap.add_argument("--kernel", default=None, help="ncu -k filter")
    a = ap.parse_args()
    cmd = ["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "cuda,sass"]
    if a.kernel:
        cmd += ["-k", a.kernel]
    out = subprocess.run(cmd, capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname, lines, hdr = None, [], None
    for r in rows:
        if r and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        elif r and r[0] == "Line No":
            hdr = r
        elif hdr and r and r[0] not in ("", "Function Name") and len(r) == len(hdr):
            try:
                lines.append((fname, int(r[0]), r[1], int(r[7] or 0), int(r[8] or 0), int(r[4] or 0)))
            except ValueError:
                pass
    tot = sum(x[3] for x in lines) or 1
    samp = sum(x[5] for x in lines) or 1
    tti = sum(x[4] for x in lines)
    print(f"warp instructions {tot:.4g}  thread instructions {tti:.4g}  SIMT efficiency {tti / tot / 32:.3f}")
    print(f"{'file':18s} {'line':>5s} {'inst%':>6s} {'simt':>5s} {'stall%':>6s}  source")
    for f, ln, src, ie, te, st in sorted(lines, key=lambda x: -x[3])[: a.top]:
        print(f"{f[:18]:18s} {ln:5d} {100 * ie / tot:6.2f} {te / max(ie, 1) / 32:5.2f} {100 * st / samp:6.2f}  {src.strip()[:90]}")


if __name__ == "__main__":
    main()
