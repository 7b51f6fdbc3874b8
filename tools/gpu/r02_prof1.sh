#!/bin/bash
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_c4_prof1.json 2> gpurun_out/bench_c4_prof1.err
tail -c 1500 gpurun_out/bench_c4_prof1.json
NOEP="--opt ep_min_frontier=2147483647"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_kernel --launch-skip 1 -c 1 -o gpurun_out/full_c4_r02a python tools/profile_step.py --config c4 --sources 4096 $NOEP > gpurun_out/ncu_c4_r02a.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o gpurun_out/full_c5ws_r02a python tools/profile_step.py --config c5ws --sources 512 $NOEP > gpurun_out/ncu_c5ws_r02a.log 2>&1
ls -la gpurun_out/*.ncu-rep
