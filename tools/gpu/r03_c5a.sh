#!/bin/bash
# c5 study, step 1: HEAD timing vs the L2 evict-first column-load build, HEAD ncu of c5ws.
mkdir -p gpurun_out/c5a
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
NOEP="ep_min_frontier=2147483647"
for lib in base colef; do
  BC_LIBBC=build/$lib/libbc.so timeout 600 python tools/ab_time.py --tag $lib --reps 2 --out gpurun_out/c5a \
     --spec c5ws:2048 --spec c5k:2048 --spec c4:4096 >> gpurun_out/c5a/ab.jsonl 2>>gpurun_out/c5a/err.log
done
BC_LIBBC=build/base/libbc.so timeout 300 python tools/ab_time.py --tag base_c148 --reps 2 --out gpurun_out/c5a \
     --spec c5ws:2048:group_ctas=148 >> gpurun_out/c5a/ab.jsonl 2>>gpurun_out/c5a/err.log
timeout 300 python tools/trace_levels.py --config c5ws --n 2 > gpurun_out/c5a/trace_c5ws.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o gpurun_out/c5a/full_c5ws_head python tools/profile_step.py --config c5ws --sources 296 --opt $NOEP > gpurun_out/c5a/ncu_c5ws.log 2>&1
cat gpurun_out/c5a/ab.jsonl | cut -c1-300
