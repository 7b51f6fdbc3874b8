#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over the late-round-2 paths: the
# per-source engine with backward push on every level that qualifies (BC_BPUSH=1), and the
# group engine's thin-row passes (BC_GROUP_MODE=2).  Logs: gpurun_out/sanitize3/.
mkdir -p gpurun_out/sanitize3
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
for tool in memcheck racecheck synccheck; do
  for graph in c1 lat64; do
    for engine in per_source_push group_thin; do
      log=gpurun_out/sanitize3/${tool}_${graph}_${engine}.log
      extra=""; stride=8
      [ $tool = racecheck ] && extra="--racecheck-report all"
      if [ $engine = per_source_push ]; then eng=per_source; envv="BC_BPUSH=1"; else eng=group; envv="BC_GROUP_MODE=2"; fi
      [ $tool = racecheck ] && [ $eng = group ] && stride=256
      env $envv timeout 900 compute-sanitizer --tool $tool $extra --error-exitcode 99 --target-processes all \
        python tools/sanitize_run.py --graph $graph --engine $eng --stride $stride > $log 2>&1
      echo "rc=$?" >> $log
      echo "$tool $graph $engine: $(tail -1 $log) $(grep 'ERROR SUMMARY\|RACECHECK SUMMARY' $log | tail -1)" | tee -a gpurun_out/sanitize3/SUMMARY.txt
    done
  done
done
