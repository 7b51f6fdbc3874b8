#!/bin/bash
# Thin rows with dynamic (group-wide claimed) level passes vs static ownership: parity, kernel ms, barrier wait.
mkdir -p gpurun_out/dyn
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_thin.py -x -q > gpurun_out/dyn/tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/dyn/tests.log
tail -3 gpurun_out/dyn/tests.log
run() {  # tag lib mode specs...
  local tag=$1 lib=$2 mode=$3; shift 3
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/dyn $a >> gpurun_out/dyn/ab.jsonl 2>>gpurun_out/dyn/err.log
}
for rep in 1 2; do
run static build/static/libbc.so 2 c5ws:2048
run dyn build/dyn/libbc.so 2 c5ws:2048
done
run dyn_c148 build/dyn/libbc.so 2 c5ws:2048:group_ctas=148
run dyn_c296 build/dyn/libbc.so 2 c5ws:2048:group_ctas=296
run dyn_c37 build/dyn/libbc.so 2 c5ws:2048:group_ctas=37
run dyn_c5k build/dyn/libbc.so 2 c5k:2048
run dyn_c4 build/dyn/libbc.so 2 c4:4096:engine=3
python - <<'PY'
import json
for l in open("gpurun_out/dyn/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        share = r["group_wait_cycles"] / (r["kernel_ms"] * 1.965e6 * 296)
        print(f"{r['tag']:9s} {r['config']:5s} mode {r['group_mode']} G {r['inflight']:3d} {r['kernel_ms']:8.1f} ms {r['gteps']:5.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc wait {share:.3f}")
PY
