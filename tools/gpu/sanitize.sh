#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over every engine on c1 and a 64x64
# lattice (race detection).  Logs: gpurun_out/sanitize/<tool>_<graph>_<engine>.log
mkdir -p gpurun_out/sanitize
for tool in memcheck racecheck synccheck; do
  for graph in c1 lat64; do
    for engine in per_source group group_fast batched; do
      log=gpurun_out/sanitize/${tool}_${graph}_${engine}.log
      extra=""; stride=8
      [ $tool = racecheck ] && extra="--racecheck-report all"
      # racecheck instruments every shared access of the group engine's 126-level sweeps:
      # 16 lattice sources keep it within the timeout (512 took > 15 min)
      eng=$engine; envv=""
      # group_fast: the group engine with the fast path forced (auto only on relabelled graphs)
      [ $engine = group_fast ] && { eng=group; envv="BC_GROUP_FAST=1"; }
      [ $engine = group ] && envv="BC_GROUP_FAST=0"
      [ $tool = racecheck ] && [ $eng = group ] && stride=256
      env $envv timeout 900 compute-sanitizer --tool $tool $extra --error-exitcode 99 --target-processes all \
        python tools/sanitize_run.py --graph $graph --engine $eng --stride $stride > $log 2>&1
      echo "rc=$?" >> $log
      echo "$tool $graph $engine: $(tail -1 $log) $(grep -c 'ERROR SUMMARY' $log) $(grep 'ERROR SUMMARY\|RACECHECK SUMMARY' $log | tail -1)"
    done
  done
done
