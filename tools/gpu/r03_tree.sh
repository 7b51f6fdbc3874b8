#!/bin/bash
# Tree-added quads (one dependent DADD per quad) vs the serial chain (build/notree): parity, kernel ms.
mkdir -p gpurun_out/tree
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
run() {  # tag lib specs...
  local tag=$1 lib=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib timeout 900 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/tree $a >> gpurun_out/tree/ab.jsonl 2>>gpurun_out/tree/err.log
}
for rep in 1 2; do
run notree build/notree/libbc.so c4:16384 c3:8192 c2d:0 c2:0 c5ws:2048 c5k:2048
run tree paper_conf_sc_mclaughlinb14_b200/libbc.so c4:16384 c3:8192 c2d:0 c2:0 c5ws:2048 c5k:2048
done
python - <<'PY'
import json
for l in open("gpurun_out/tree/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); pc = r["phase_cycles"]
        print(f"{r['tag']:7s} {r['config']:5s} k={r['sources']:6d} {r['kernel_ms']:8.1f} ms {r['gteps']:6.1f} GTEPS fwd {pc[0]/1e9:6.2f} bwd {pc[2]/1e9:6.2f}")
PY
for c in c4_16384 c3_8192 c2d_0 c2_0; do f=$(ls gpurun_out/tree/tree_${c}_*.npy | head -1); b=${f/tree_/notree_}; python tools/ab_time.py --compare $f $b; done
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bpush.py tests/test_gpu_thin.py tests/test_gpu_random_graphs.py -x -q > gpurun_out/tree/tests.log 2>&1
echo "tests rc=$?"; tail -2 gpurun_out/tree/tests.log
