#!/bin/bash
# Thin rows, push forward: parity (thin tests on the default build), then kernel ms of variants.
mkdir -p gpurun_out/push
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_thin.py -x -q > gpurun_out/push/tests.log 2>&1
echo "thin tests rc=$?" >> gpurun_out/push/tests.log
tail -3 gpurun_out/push/tests.log
run() {  # tag lib mode specs...
  local tag=$1 lib=$2 mode=$3; shift 3
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/push $a >> gpurun_out/push/ab.jsonl 2>>gpurun_out/push/err.log
}
run base build/base/libbc.so -1 c5ws:2048
for v in push_u4 push_u3 push_u2 push_u6 pull_u4 push_vw2u3; do run $v build/$v/libbc.so 2 c5ws:2048; done
run push_u4_c5k build/push_u4/libbc.so 2 c5k:2048
python - <<'PY'
import json
for l in open("gpurun_out/push/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:12s} {r['config']:5s} {r['kernel_ms']:8.1f} ms {r['gteps']:5.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc")
PY
