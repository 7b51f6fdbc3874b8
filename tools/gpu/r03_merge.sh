#!/bin/bash
# Alg. 5 with the B200 guard in one launch (sampling sources + the rest) vs two launches
# (BC_NO_MERGE=1): parity subsets, kernel ms, bench lines of c1 and c4.
M=gpurun_out/merge
mkdir -p $M
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_group.py tests/test_gpu_scale.py tests/test_gpu_thin.py -x -q > $M/tests.log 2>&1
echo "tests rc=$?"; tail -2 $M/tests.log
run() {  # tag env specs...
  local tag=$1 envv=$2; shift 2
  local a=""; for s in "$@"; do a="$a --spec $s"; done
  env $envv timeout 900 python tools/ab_time.py --tag $tag --reps 3 --out $M $a >> $M/ab.jsonl 2>>$M/err.log
}
run two "BC_NO_MERGE=1" c1:0 c2d:0 c3:8192 c4:16384 c5ws:2048 c5k:2048
run one "X=1" c1:0 c2d:0 c3:8192 c4:16384 c5ws:2048 c5k:2048
python - <<'PY'
import json
for l in open("gpurun_out/merge/ab.jsonl"):
    if l.startswith("{"):
        r = json.loads(l)
        print(f"{r['tag']:4s} {r['config']:5s} k={r['sources']:6d} {r['kernel_ms']:9.3f} ms {r['gteps']:6.1f} GTEPS")
PY
for c in c1_0 c2d_0 c3_8192 c4_16384; do f=$(ls $M/one_${c}_*.npy | head -1); b=${f/one_/two_}; python tools/ab_time.py --compare $f $b; done
timeout 600 python bench.py --config c1 --steps 20 > $M/bench_c1.json 2> $M/bench_c1.err; echo "c1: $(head -c 200 $M/bench_c1.json)"
timeout 900 python bench.py --steps 20 --warmup 5 > $M/bench_c4.json 2> $M/bench_c4.err; echo "c4: $(head -c 200 $M/bench_c4.json)"
