#!/bin/bash
# Backward successor extraction (four successors per window scan) in the group engine
# (thin rows on c5ws, fast path on c5k): parity, kernel ms vs build/noext; c4 block size /
# L2 window re-sweep after the backward push.
mkdir -p gpurun_out/ext
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_thin.py tests/test_gpu_group.py tests/test_gpu_random_graphs.py -x -q > gpurun_out/ext/tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/ext/tests.log
tail -3 gpurun_out/ext/tests.log
run() {  # tag lib specs...
  local tag=$1 lib=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib timeout 900 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/ext $a >> gpurun_out/ext/ab.jsonl 2>>gpurun_out/ext/err.log
}
for rep in 1 2; do
run noext build/noext/libbc.so c5ws:2048 c5k:2048
run ext paper_conf_sc_mclaughlinb14_b200/libbc.so c5ws:2048 c5k:2048
done
run c4knob paper_conf_sc_mclaughlinb14_b200/libbc.so c4:16384 c4:16384:block_threads=1024 c4:16384:l2_persist=-1 c4:16384:block_threads=1024,l2_persist=-1 c4:16384 c4:16384:block_threads=1024 c4:16384:block_threads=1024,l2_persist=-1 c3:8192:l2_persist=-1 c2d:0:l2_persist=-1 c3:8192 c2d:0
python - <<'PY'
import json
for l in open("gpurun_out/ext/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        o = {k: v for k, v in r["opts"].items() if k not in ("strategy", "ep_min_frontier")}
        print(f"{r['tag']:7s} {r['config']:5s} k={r['sources']:6d} {str(o):45s} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f}")
PY
