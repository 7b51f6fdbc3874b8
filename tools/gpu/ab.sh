#!/bin/bash
# A/B of the working tree against a baseline build (build/base/libbc.so, built from an
# earlier commit and shipped with the snapshot).  SPECS: config:sources[:opts] list.
mkdir -p gpurun_out/ab
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
SPECS=${SPECS:-"c4:16384 c3:8192 c2d:0 c2:0 c1:0"}
args=""; for s in $SPECS; do args="$args --spec $s"; done
for round in 1 2; do
  BC_LIBBC=build/base/libbc.so timeout 900 python tools/ab_time.py --tag base $args >> gpurun_out/ab/base.jsonl 2>>gpurun_out/ab/err.log
  timeout 900 python tools/ab_time.py --tag new $args >> gpurun_out/ab/new.jsonl 2>>gpurun_out/ab/err.log
done
python - <<'PY'
import json, collections, subprocess
rows = [json.loads(l) for f in ("gpurun_out/ab/base.jsonl", "gpurun_out/ab/new.jsonl") for l in open(f) if l.startswith("{")]
best = collections.defaultdict(dict)
for r in rows:
    key = (r["config"], r["sources"], json.dumps(r["opts"], sort_keys=True))
    b = best[key].get(r["tag"])
    if b is None or r["kernel_ms"] < b["kernel_ms"]:
        best[key][r["tag"]] = r
for key, d in best.items():
    if "base" in d and "new" in d:
        x, y = d["base"], d["new"]
        cmp = subprocess.run(["python", "tools/ab_time.py", "--compare", f"gpurun_out/ab/{y['file']}.npy", f"gpurun_out/ab/{x['file']}.npy"], capture_output=True, text=True).stdout.strip()
        print(f"{key[0]:5s} k={key[1]:6d} base {x['kernel_ms']:9.2f} ms  new {y['kernel_ms']:9.2f} ms  speedup {x['kernel_ms']/y['kernel_ms']:.3f}  new GTEPS {y['gteps']:.1f}  {cmp}")
PY
