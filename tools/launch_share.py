#!/usr/bin/env python
"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv --log-file X):
per kernel name the number of launches, total device time and share of the total.

    python tools/launch_share.py gpurun_out/launches_c4.csv [--out profiles/r01/launches_c4_summary.txt]
"""
import argparse
import collections
import csv
import io


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--out")
    a = ap.parse_args()
    text = open(a.csv).read()
    start = text.find('"ID"')
    rows = list(csv.reader(io.StringIO(text[start:])))
    h = rows[0]
    ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    tot = collections.Counter()
    cnt = collections.Counter()
    scale = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0,
             "second": 1e3, "s": 1e3}
    for r in rows[1:]:
        if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0]
        ms = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
        tot[name] += ms
        cnt[name] += 1
    all_ms = sum(tot.values()) or 1.0
    lines = [f"{'kernel':60s} {'launches':>8s} {'total ms':>12s} {'share':>7s}"]
    for k, v in tot.most_common():
        lines.append(f"{k[:60]:60s} {cnt[k]:8d} {v:12.3f} {100 * v / all_ms:6.2f}%")
    lines.append(f"{'(all)':60s} {sum(cnt.values()):8d} {all_ms:12.3f}")
    out = "\n".join(lines)
    print(out)
    if a.out:
        open(a.out, "w").write(out + "\n")


if __name__ == "__main__":
    main()
