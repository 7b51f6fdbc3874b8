#!/bin/bash
# Round-2 final measurement pass (one B200): bench lines of every config at HEAD (with the
# L2 fields from profiles/traffic.json), the ncu launch list of the default bench command,
# the reference arm, the multi-GPU refusal on a 1-GPU box, smoke().
mkdir -p gpurun_out/final
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/final/bench_c4.json 2> gpurun_out/final/bench_c4.err
echo "c4: $(head -c 250 gpurun_out/final/bench_c4.json)"
for spec in "c1 0 20" "c2 0 5" "c2d 0 5" "c3 0 5" "c5ws 8192 3" "c5k 8192 3"; do
  set -- $spec
  src=""; [ "$2" != 0 ] && src="--sources $2"
  timeout 1500 python bench.py --config $1 $src --steps $3 > gpurun_out/final/bench_$1.json 2> gpurun_out/final/bench_$1.err
  echo "$1: $(head -c 250 gpurun_out/final/bench_$1.json)"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches_c4.csv python bench.py --no-cpu-baseline --steps 2 --warmup 3 > gpurun_out/final/bench_c4_under_ncu.json 2>/dev/null
echo "ncu rc=$?"
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/final/reference.json 2> gpurun_out/final/reference.err
echo "reference: $(head -c 300 gpurun_out/final/reference.json)"
timeout 120 python bench.py --gpus 2 > gpurun_out/final/gpus2.out 2> gpurun_out/final/gpus2.err; echo "gpus2 rc=$?"; tail -2 gpurun_out/final/gpus2.err
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/final/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/final/smoke.log
