#!/bin/bash
# Kernel-time A/B of several library builds: LIBS="tag:path ..." (path "default" = the tree's
# libbc.so), SPECS as in tools/ab_time.py.  Prints min kernel ms per (spec, tag).
mkdir -p gpurun_out/abm
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
args=""; for s in $SPECS; do args="$args --spec $s"; done
for round in 1 2; do
  for spec in $LIBS; do
    tag=${spec%%:*}; lib=${spec#*:}
    if [ "$lib" = default ]; then
      timeout 900 python tools/ab_time.py --tag $tag --out gpurun_out/abm $args >> gpurun_out/abm/all.jsonl 2>>gpurun_out/abm/err.log
    else
      BC_LIBBC=$lib timeout 900 python tools/ab_time.py --tag $tag --out gpurun_out/abm $args >> gpurun_out/abm/all.jsonl 2>>gpurun_out/abm/err.log
    fi
  done
done
python - <<'PY'
import json, collections
rows = [json.loads(l) for l in open("gpurun_out/abm/all.jsonl") if l.startswith("{")]
best = collections.defaultdict(dict)
for r in rows:
    key = (r["config"], r["sources"], json.dumps(r["opts"], sort_keys=True))
    b = best[key].get(r["tag"])
    if b is None or r["kernel_ms"] < b["kernel_ms"]:
        best[key][r["tag"]] = r
for key, d in best.items():
    print(key[0], key[1], key[2])
    for tag, r in sorted(d.items(), key=lambda x: x[1]["kernel_ms"]):
        print(f"   {tag:10s} {r['kernel_ms']:9.2f} ms  {r['gteps']:7.2f} GTEPS  phase_cycles {r['phase_cycles']}")
PY
