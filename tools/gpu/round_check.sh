#!/bin/bash
# Round check (gpurun): build, all GPU tests, bench lines (c4 default + bounded c5), the ncu
# launch list of the default bench command, DRAM traffic per config (profiles/traffic.json)
# and full captures of the main c4 launch and of the c5k group kernel.
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gputests.log
timeout 600 python bench.py > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 600 python bench.py --config c5ws --sources 8192 > gpurun_out/bench_c5ws.json 2> gpurun_out/bench_c5ws.err
timeout 900 python bench.py --config c5k --sources 8192 > gpurun_out/bench_c5k.json 2> gpurun_out/bench_c5k.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --no-cpu-baseline > gpurun_out/bench_c4_under_ncu.json 2>/dev/null
NOEP="--opt ep_min_frontier=2147483647"
for spec in "c4 16384" "c5ws 2048" "c5k 2048"; do
  set -- $spec
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"bc_kernel|group_kernel" -o gpurun_out/traffic_$1 python tools/profile_step.py --config $1 --sources $2 $NOEP --stats-out gpurun_out/stats_$1.json > gpurun_out/traffic_$1.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_kernel --launch-skip 1 -c 1 -o gpurun_out/full_c4_main python tools/profile_step.py --config c4 --sources 4096 $NOEP > gpurun_out/ncu_full_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o gpurun_out/full_c5k_group python tools/profile_step.py --config c5k --sources 512 $NOEP > gpurun_out/ncu_full_c5k.log 2>&1
