#!/bin/bash
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_c4_check2.json 2> gpurun_out/bench_c4_check2.err
head -c 400 gpurun_out/bench_c4_check2.json; echo
LIBS="new:default" SPECS="c4:4096:strategy=we c4:4096:strategy=hybrid c4:4096:strategy=sampling,ep_min_frontier=512 c3:4096:strategy=we c3:4096:strategy=hybrid c3:4096:strategy=sampling,ep_min_frontier=512 c2:16384:strategy=we c2:16384:strategy=hybrid c2:16384:strategy=sampling,ep_min_frontier=512 c2d:16384:strategy=we c2d:16384:strategy=hybrid c2d:16384:strategy=sampling,ep_min_frontier=512" bash tools/gpu/ab_multi.sh > gpurun_out/abm_sel.txt 2>&1
cat gpurun_out/abm_sel.txt
rm -rf gpurun_out/abm
timeout 2400 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/gputests_check2.log 2>&1; echo "tests rc=$?" >> gpurun_out/gputests_check2.log
tail -25 gpurun_out/gputests_check2.log
