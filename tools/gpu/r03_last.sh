#!/bin/bash
# Last pass at HEAD: bench lines of the remaining configs, then the whole GPU suite and smoke.
M=gpurun_out/last
mkdir -p $M
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
for spec in "c2 0 5" "c2d 0 5" "c3 0 5" "c5ws 8192 3" "c5k 8192 3"; do
  set -- $spec
  src=""; [ "$2" != 0 ] && src="--sources $2"
  timeout 1500 python bench.py --config $1 $src --steps $3 > $M/bench_$1.json 2> $M/bench_$1.err
  echo "$1: $(head -c 160 $M/bench_$1.json)"
done
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $M/smoke.log
timeout 2700 python -m pytest tests -m gpu -q > $M/gputests.log 2>&1
echo "gpu tests rc=$?"; tail -2 $M/gputests.log
