#!/usr/bin/env python
"""Per-CUDA-source-line instruction and stall shares from an ncu report (needs -lineinfo)."""
import collections
import csv
import io
import subprocess
import sys


def main(rep, top=30):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    ie = hdr.index("Instructions Executed")
    ist = hdr.index("Warp Stall Sampling (All Samples)")
    ex, st, src = collections.Counter(), collections.Counter(), {}
    cur, fname = ("?", 0), "?"
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] in ("Function Name", "Line No"):
            continue
        if r[0]:
            cur = (fname, int(r[0]))
            src[cur] = r[1]
            continue
        try:
            ex[cur] += float(r[ie] or 0)
            st[cur] += float(r[ist] or 0)
        except (ValueError, IndexError):
            pass
    te, ts = sum(ex.values()) or 1, sum(st.values()) or 1
    print(f"{'file':16s} {'line':>5s} {'exec%':>7s} {'stall%':>7s}  source")
    for k, _ in sorted(st.items(), key=lambda x: -x[1])[:top]:
        print(f"{k[0][:16]:16s} {k[1]:5d} {100 * ex[k] / te:7.2f} {100 * st[k] / ts:7.2f}  {src.get(k, '?').strip()[:90]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
