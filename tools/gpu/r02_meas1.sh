#!/bin/bash
# Round-2 measurement pass: N1 ablation at HEAD, c5 level traces, per-config bench lines,
# ncu DRAM + L2 traffic of every config's traversal launches (profiles/traffic.json).
mkdir -p gpurun_out/meas
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1500 python tools/ablation.py --configs c1,c2,c2d,c3,c4,c5ws,c5k --sweep-configs c2,c3,c4,c5ws,c5k --out gpurun_out/meas/ablation_r02.json > gpurun_out/meas/ablation.log 2>&1
echo "ablation rc=$?"
for c in c5ws c5k; do timeout 300 python tools/trace_levels.py --config $c --n 2 > gpurun_out/meas/trace_$c.txt 2>&1; done
NOEP="--opt ep_min_frontier=2147483647"
for spec in "c1 0" "c2 0" "c2d 0" "c3 0" "c4 0" "c5ws 2048" "c5k 2048"; do
  set -- $spec
  src=""; [ "$2" != 0 ] && src="--sources $2"
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,gpu__time_duration.sum --clock-control none -k regex:"bc_kernel|group_kernel" -o gpurun_out/meas/traffic_$1 python tools/profile_step.py --config $1 $src $NOEP --stats-out gpurun_out/meas/stats_$1.json > gpurun_out/meas/traffic_$1.log 2>&1
  python tools/make_traffic.py gpurun_out/meas/traffic_$1.ncu-rep gpurun_out/meas/stats_$1.json --out gpurun_out/meas/traffic.json >> gpurun_out/meas/make_traffic.log 2>&1
done
cat gpurun_out/meas/make_traffic.log
for spec in "c1 0 10" "c2 0 5" "c2d 0 5" "c3 0 5" "c5ws 8192 3" "c5k 8192 3"; do
  set -- $spec
  src=""; [ "$2" != 0 ] && src="--sources $2"
  timeout 1200 python bench.py --config $1 $src --steps $3 > gpurun_out/meas/bench_$1.json 2> gpurun_out/meas/bench_$1.err
  echo "$1: $(head -c 300 gpurun_out/meas/bench_$1.json)"
done
