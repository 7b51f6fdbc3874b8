#!/bin/bash
# Knob re-sweep on c4 after the backward push (kernel ms, 16,384 sources; 2 reps each).
mkdir -p gpurun_out/knobs
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag env specs...
  local tag=$1 envv=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  env $envv timeout 900 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/knobs $a >> gpurun_out/knobs/ab.jsonl 2>>gpurun_out/knobs/err.log
}
run default "X=1" c4:16384 c4:16384:seq_max_deg=64 c4:16384:seq_max_deg=256 c4:16384:warp_max_deg=4096 c4:16384:warp_max_deg=16384 c4:16384:block_threads=1024 c4:16384:l2_persist=-1 c4:16384:inflight=148
run bp3 "BC_BPUSH=3" c4:16384
run bp2b "BC_BPUSH=2" c4:16384
run c3seq "X=1" c3:8192:seq_max_deg=64 c3:8192:seq_max_deg=32 c3:8192:block_threads=1024 c3:8192:block_threads=256
run c3 "X=1" c3:8192 c2d:0 c2d:0:seq_max_deg=32 c2d:0:block_threads=256
python - <<'PY'
import json
for l in open("gpurun_out/knobs/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        o = {k: v for k, v in r["opts"].items() if k not in ("strategy", "ep_min_frontier")}
        print(f"{r['tag']:8s} {r['config']:5s} k={r['sources']:6d} {str(o):40s} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f}")
PY
