#!/bin/bash
# A/B of library variants (gpurun): VARIANTS="minb3:-DBC_MINB512=3 ..." built with
# `make variant`, each timed on the lines of $SWEEP against the default build.
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
for spec in $VARIANTS; do
  name=${spec%%:*}; flags=${spec#*:}
  make variant VARIANT=$name VFLAGS="${flags//,/ }" >> gpurun_out/make.log 2>&1 || echo "variant $name failed" >> gpurun_out/variants.log
done
LIST=${SWEEP:-tools/gpu/sweep_default.txt}
for spec in default $VARIANTS; do
  name=${spec%%:*}
  lib=""; [ "$name" != default ] && lib=build/$name/libbc.so
  while read -r cfg n rest; do
    [ -z "$cfg" ] && continue
    case "$cfg" in \#*) continue;; esac
    o=""; for x in $rest; do o="$o --opt $x"; done
    echo "== [$name] $cfg n=$n $rest" >> gpurun_out/variants.log
    env ${lib:+BC_LIBBC=$lib} timeout 300 python tools/profile_step.py --config $cfg --sources $n --repeat 2 $o --opt ep_min_frontier=2147483647 2>&1 | tail -n 1 >> gpurun_out/variants.log
  done < $LIST
done
