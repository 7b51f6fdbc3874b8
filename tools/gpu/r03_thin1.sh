#!/bin/bash
# Thin-row group passes: parity first, then kernel ms against HEAD (build/base) and variants.
mkdir -p gpurun_out/thin1
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_thin.py -x -q > gpurun_out/thin1/tests.log 2>&1
echo "thin tests rc=$?" >> gpurun_out/thin1/tests.log
tail -5 gpurun_out/thin1/tests.log
run() {  # tag lib mode specs...
  local tag=$1 lib=$2 mode=$3; shift 3
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  BC_LIBBC=$lib BC_GROUP_MODE=$mode timeout 600 python tools/ab_time.py --tag $tag --reps 2 --out gpurun_out/thin1 $a >> gpurun_out/thin1/ab.jsonl 2>>gpurun_out/thin1/err.log
}
run base build/base/libbc.so -1 c5ws:2048
run thin paper_conf_sc_mclaughlinb14_b200/libbc.so 2 c5ws:2048
run thin_vw8u2 build/thinvw8u2/libbc.so 2 c5ws:2048
run thin_vw4u2 build/thinvw4u2/libbc.so 2 c5ws:2048
run thin_c148 paper_conf_sc_mclaughlinb14_b200/libbc.so 2 c5ws:2048:group_ctas=148
run thin_c37 paper_conf_sc_mclaughlinb14_b200/libbc.so 2 c5ws:2048:group_ctas=37
run thin_c5k paper_conf_sc_mclaughlinb14_b200/libbc.so 2 c5k:2048
python - <<'PY'
import json
for l in open("gpurun_out/thin1/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l); print(f"{r['tag']:12s} {r['config']:5s} {r['sources']:6d} {r['kernel_ms']:9.1f} ms {r['gteps']:6.1f} GTEPS arcs {r['arcs_scanned']}")
PY
