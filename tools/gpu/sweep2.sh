#!/bin/bash
# Kernel-ms sweep (gpurun): lines "cfg nsrc opt=val ..." from $SWEEP (or the default list).
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
LIST=${SWEEP:-tools/gpu/sweep_default.txt}
while read -r cfg n rest; do
  [ -z "$cfg" ] && continue
  case "$cfg" in \#*) continue;; esac
  o=""; for x in $rest; do o="$o --opt $x"; done
  echo "== $cfg n=$n $rest" >> gpurun_out/sweep2.log
  timeout 300 python tools/profile_step.py --config $cfg --sources $n --repeat 2 $o --opt ep_min_frontier=2147483647 2>&1 | tail -n 1 >> gpurun_out/sweep2.log || echo "FAILED" >> gpurun_out/sweep2.log
done < $LIST
