#!/bin/bash
# Thin-row passes: virtual-warp width / arcs in flight, forward and backward (kernel ms, c5ws 2,048 sources).
mkdir -p gpurun_out/thin2
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag lib mode specs...
  local tag=$1 lib=$2 mode=$3; shift 3
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/thin2 $a >> gpurun_out/thin2/ab.jsonl 2>>gpurun_out/thin2/err.log
}
run base build/base/libbc.so -1 c5ws:2048
for v in f4u3b1u4 f1u4b1u4 f2u5b1u4 f1u6b1u6 f4u3b2u3 f2u3b1u3 f4u3b1u2; do run $v build/$v/libbc.so 2 c5ws:2048; done
python - <<'PY'
import json
for l in open("gpurun_out/thin2/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:10s} {r['config']:5s} {r['kernel_ms']:8.1f} ms {r['gteps']:5.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc")
PY
