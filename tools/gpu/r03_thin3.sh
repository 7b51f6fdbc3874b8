#!/bin/bash
# Thin-row passes: virtual-warp width / arcs in flight, forward and backward (kernel ms, c5ws 2,048 sources).
mkdir -p gpurun_out/thin3
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag lib mode specs...
  local tag=$1 lib=$2 mode=$3; shift 3
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/thin3 $a >> gpurun_out/thin3/ab.jsonl 2>>gpurun_out/thin3/err.log
}
run base build/base/libbc.so -1 c5ws:2048
for v in pf_f1u4b1u4 nopf_f1u4b1u4 pf_f1u3b1u3 pf_f1u2b1u4 pf_f1u4b1u2 pf_f1u5b1u5; do run $v build/$v/libbc.so 2 c5ws:2048; done
run pf_c148 build/pf_f1u4b1u4/libbc.so 2 c5ws:2048:group_ctas=148
run pf_c37 build/pf_f1u4b1u4/libbc.so 2 c5ws:2048:group_ctas=37
run pf_c5k build/pf_f1u4b1u4/libbc.so 2 c5k:2048
run base_c5k build/base/libbc.so -1 c5k:2048
python - <<'PY'
import json
for l in open("gpurun_out/thin3/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:10s} {r['config']:5s} {r['kernel_ms']:8.1f} ms {r['gteps']:5.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc")
PY
