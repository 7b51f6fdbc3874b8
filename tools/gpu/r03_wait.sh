#!/bin/bash
# Group barrier wait share per level pass kind (generic / fast / thin), and thin parity at HEAD.
mkdir -p gpurun_out/wait
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_thin.py tests/test_gpu_group.py -x -q > gpurun_out/wait/tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/wait/tests.log
tail -3 gpurun_out/wait/tests.log
run() {  # tag mode specs...
  local tag=$1 mode=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/wait $a >> gpurun_out/wait/ab.jsonl 2>>gpurun_out/wait/err.log
}
run generic 0 c5ws:2048 c5k:2048
run fast 1 c5ws:2048 c5k:2048
run thin 2 c5ws:2048
python - <<'PY'
import json
for l in open("gpurun_out/wait/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        grid = 296
        share = r["group_wait_cycles"] / (r["kernel_ms"] * 1.965e6 * grid)
        print(f"{r['tag']:8s} {r['config']:5s} mode {r['group_mode']} G {r['inflight']:3d} {r['kernel_ms']:8.1f} ms {r['gteps']:5.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc  barrier-wait share {share:.3f}")
PY
