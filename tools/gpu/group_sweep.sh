#!/bin/bash
# Group-engine check + sweep (gpurun): parity tests, then kernel ms per config / group size.
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_group.py -x -q > gpurun_out/group_tests.log 2>&1
echo "group tests rc=$?" >> gpurun_out/group_tests.log
run() {  # cfg sources opts...
  local cfg=$1 n=$2; shift 2
  local o=""; for x in "$@"; do o="$o --opt $x"; done
  echo "== $cfg n=$n $*" >> gpurun_out/sweep.log
  timeout 300 python tools/profile_step.py --config $cfg --sources $n --repeat 2 $o --opt ep_min_frontier=2147483647 >> gpurun_out/sweep.log 2>&1 || echo "FAILED rc=$?" >> gpurun_out/sweep.log
}
for c in 0 148 74 37; do run c5ws 2048 engine=3 group_ctas=$c; done
for c in 0 148 74 37; do run c5k 2048 engine=3 group_ctas=$c; done
run c4 16384 engine=1
for c in 0 4 9 18 37; do run c4 16384 engine=3 group_ctas=$c; done
