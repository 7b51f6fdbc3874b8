#!/bin/bash
# Backward push: its parity tests + group engine tests, then group fast path (c5k) timing per ratio.
mkdir -p gpurun_out/bpush2
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_bpush.py tests/test_gpu_group.py -x -q > gpurun_out/bpush2/tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/bpush2/tests.log
tail -3 gpurun_out/bpush2/tests.log
run() {  # tag bpush specs...
  local tag=$1 bp=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_BPUSH=$bp timeout 900 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/bpush2 $a >> gpurun_out/bpush2/ab.jsonl 2>>gpurun_out/bpush2/err.log
}
for bp in 0 1 2 4; do run bp$bp $bp c5k:2048; done
run bp0 0 c4:16384
run bp2 2 c4:16384
python - <<'PY'
import json
for l in open("gpurun_out/bpush2/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:5s} {r['config']:5s} k={r['sources']:6d} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc scanned {r['arcs_scanned']/r['sources']/1e6:6.2f} M/src mode {r.get('group_mode')}")
PY
