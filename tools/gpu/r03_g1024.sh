#!/bin/bash
# Group engine with 1,024-thread CTAs (tuning build build/g1024, BC_GROUP_NT=1024) vs 512.
mkdir -p gpurun_out/g1024
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag env specs...
  local tag=$1 envv=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  env $envv timeout 900 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/g1024 $a >> gpurun_out/g1024/ab.jsonl 2>>gpurun_out/g1024/err.log
}
run nt512 "BC_LIBBC=build/g1024/libbc.so" c5ws:2048 c5k:2048
run nt1024 "BC_LIBBC=build/g1024/libbc.so BC_GROUP_NT=1024" c5ws:2048 c5ws:2048:group_ctas=74 c5k:2048 c5k:2048:group_ctas=9 c5k:2048:group_ctas=6
BC_LIBBC=build/g1024/libbc.so BC_GROUP_NT=1024 BC_GROUP_MODE=2 timeout 600 python -m pytest tests/test_gpu_thin.py -x -q -k "c5 or c1_exact" > gpurun_out/g1024/tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/g1024/tests.log
python - <<'PY'
import json
for l in open("gpurun_out/g1024/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        o = {k: v for k, v in r["opts"].items() if k not in ("strategy", "ep_min_frontier")}
        print(f"{r['tag']:7s} {r['config']:5s} k={r['sources']:6d} {str(o):25s} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} G {r['inflight']}")
PY
