#!/bin/bash
# c4 with the auto 1,024-thread CTAs and no persisting-L2 window (skewed graph, shared-memory
# codes): parity at scale, bench line, launch list, full ncu of the main launch.
M=gpurun_out/c4b
mkdir -p $M
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_scale.py tests/test_gpu_parity.py tests/test_gpu_bpush.py -x -q > $M/tests.log 2>&1
echo "tests rc=$?" >> $M/tests.log; tail -3 $M/tests.log
timeout 900 python bench.py --steps 20 --warmup 5 > $M/bench_c4.json 2> $M/bench_c4.err
echo "c4: $(head -c 300 $M/bench_c4.json)"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches_c4.csv python bench.py --no-cpu-baseline --steps 2 --warmup 3 > $M/bench_c4_under_ncu.json 2>/dev/null
echo "ncu launches rc=$?"
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,gpu__time_duration.sum --clock-control none -k regex:"bc_kernel" -o $M/traffic_c4 python tools/profile_step.py --config c4 --opt ep_min_frontier=2147483647 --stats-out $M/stats_c4.json > $M/traffic_c4.log 2>&1
python tools/make_traffic.py $M/traffic_c4.ncu-rep $M/stats_c4.json --out $M/traffic.json > $M/make_traffic.log 2>&1; tail -1 $M/make_traffic.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_kernel --launch-skip 1 -c 1 -o $M/full_c4 python tools/profile_step.py --config c4 --sources 4096 --opt ep_min_frontier=2147483647 > $M/ncu_c4.log 2>&1
echo "ncu c4 rc=$?"
