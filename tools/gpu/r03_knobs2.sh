#!/bin/bash
# Knob re-sweep at HEAD (kernel ms): c4 push ratio / row split at 1,024 threads, c5k group size, c5ws group size.
mkdir -p gpurun_out/knobs2
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag env specs...
  local tag=$1 envv=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  env $envv timeout 900 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/knobs2 $a >> gpurun_out/knobs2/ab.jsonl 2>>gpurun_out/knobs2/err.log
}
run c4 "X=1" c4:16384 c4:16384:seq_max_deg=64 c4:16384:seq_max_deg=256 c4:16384:warp_max_deg=16384 c4:16384:warp_max_deg=2048
run bp1 "BC_BPUSH=1" c4:16384
run bp3 "BC_BPUSH=3" c4:16384
run c5 "X=1" c5k:2048 c5k:2048:group_ctas=12 c5k:2048:group_ctas=24 c5k:2048:group_ctas=37 c5ws:2048 c5ws:2048:group_ctas=148 c5ws:2048:group_ctas=49
python - <<'PY'
import json
for l in open("gpurun_out/knobs2/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        o = {k: v for k, v in r["opts"].items() if k not in ("strategy", "ep_min_frontier")}
        print(f"{r['tag']:5s} {r['config']:5s} k={r['sources']:6d} {str(o):32s} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} G {r['inflight']}")
PY
