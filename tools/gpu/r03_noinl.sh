#!/bin/bash
# Thin rows: inlined vs out-of-line level passes (register pressure), kernel ms c5ws; ncu of the best.
mkdir -p gpurun_out/noinl
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag lib mode specs...
  local tag=$1 lib=$2 mode=$3; shift 3
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/noinl $a >> gpurun_out/noinl/ab.jsonl 2>>gpurun_out/noinl/err.log
}
for rep in 1 2; do
run base build/base/libbc.so -1 c5ws:2048
for v in inl_u4 noinl_u4 noinl_u6 noinl_u4_nopf; do run $v build/$v/libbc.so 2 c5ws:2048; done
done
python - <<'PY'
import json
for l in open("gpurun_out/noinl/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:14s} {r['config']:5s} {r['kernel_ms']:8.1f} ms {r['gteps']:5.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f} Gcyc")
PY
BC_LIBBC=build/noinl_u4/libbc.so BC_GROUP_MODE=2 timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o gpurun_out/noinl/full_c5ws_thin python tools/profile_step.py --config c5ws --sources 296 --opt ep_min_frontier=2147483647 > gpurun_out/noinl/ncu.log 2>&1
tail -2 gpurun_out/noinl/ncu.log
