#!/bin/bash
# Backward push for levels whose next level has fewer arcs (fast path, per-source engine):
# parity (whole GPU suite), then kernel ms per push ratio.
mkdir -p gpurun_out/bpush
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/bpush/tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/bpush/tests.log
tail -3 gpurun_out/bpush/tests.log
run() {  # tag bpush specs...
  local tag=$1 bp=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_BPUSH=$bp timeout 900 python tools/ab_time.py --tag $tag --reps 3 --out gpurun_out/bpush $a >> gpurun_out/bpush/ab.jsonl 2>>gpurun_out/bpush/err.log
}
for bp in 0 1 2 4 8; do run bp$bp $bp c4:16384 c3:8192 c2d:0 c1:0; done
python - <<'PY'
import json
for l in open("gpurun_out/bpush/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:5s} {r['config']:5s} k={r['sources']:6d} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc scanned {r['arcs_scanned']/r['sources']/1e6:6.2f} M/src")
PY
for f in gpurun_out/bpush/bp4_*.npy; do b=${f/bp4_/bp0_}; python tools/ab_time.py --compare $f $b; done
