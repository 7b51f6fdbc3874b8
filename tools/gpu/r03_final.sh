#!/bin/bash
# Final round-2 pass at HEAD (one B200): N1 ablation, DRAM/L2 traffic per config, driver-style
# bench lines of every config, ncu launch list of the default bench command, full ncu captures
# (c4 main launch, c5ws and c5k group kernels), the reference arm, the 2-GPU refusal, smoke,
# and the whole GPU suite last.   BC_HEAD names the commit (no .git on the box).
M=gpurun_out/final3
mkdir -p $M
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $M/smoke.log
NOEP="--opt ep_min_frontier=2147483647"
rm -f $M/traffic.json
for spec in "c1 0" "c2 0" "c2d 0" "c3 0" "c4 0" "c5ws 2048" "c5k 2048"; do
  set -- $spec
  src=""; [ "$2" != 0 ] && src="--sources $2"
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,gpu__time_duration.sum --clock-control none -k regex:"bc_kernel|group_kernel" -o $M/traffic_$1 python tools/profile_step.py --config $1 $src $NOEP --stats-out $M/stats_$1.json > $M/traffic_$1.log 2>&1
  python tools/make_traffic.py $M/traffic_$1.ncu-rep $M/stats_$1.json --out $M/traffic.json >> $M/make_traffic.log 2>&1
  rm -f $M/traffic_$1.ncu-rep   # gpurun copies back <= 64 MiB: keep the numbers, not the reports
done
cp $M/traffic.json profiles/traffic.json
timeout 900 python bench.py --steps 20 --warmup 5 > $M/bench_c4.json 2> $M/bench_c4.err
echo "c4: $(head -c 200 $M/bench_c4.json)"
for spec in "c1 0 20" "c2 0 5" "c2d 0 5" "c3 0 5" "c5ws 8192 3" "c5k 8192 3"; do
  set -- $spec
  src=""; [ "$2" != 0 ] && src="--sources $2"
  timeout 1500 python bench.py --config $1 $src --steps $3 > $M/bench_$1.json 2> $M/bench_$1.err
  echo "$1: $(head -c 200 $M/bench_$1.json)"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches_c4.csv python bench.py --no-cpu-baseline --steps 2 --warmup 3 > $M/bench_c4_under_ncu.json 2>/dev/null
echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_kernel --launch-skip 1 -c 1 -o $M/full_c4 python tools/profile_step.py --config c4 --sources 4096 $NOEP > $M/ncu_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o $M/full_c5ws python tools/profile_step.py --config c5ws --sources 296 $NOEP > $M/ncu_c5ws.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o $M/full_c5k python tools/profile_step.py --config c5k --sources 64 $NOEP > $M/ncu_c5k.log 2>&1
echo "ncu full rc=$?"
for k in c4 c5ws c5k; do
  python tools/ncu_summary.py $M/full_$k.ncu-rep > $M/ncu_full_$k.txt 2>&1
  python tools/ncu_lines2.py $M/full_$k.ncu-rep > $M/ncu_full_${k}_lines.txt 2>&1
  rm -f $M/full_$k.ncu-rep
done
du -sh $M
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $M/reference.json 2> $M/reference.err
echo "reference: $(head -c 200 $M/reference.json)"
timeout 120 python bench.py --gpus 2 > $M/gpus2.out 2> $M/gpus2.err; echo "gpus2 rc=$?"; tail -1 $M/gpus2.err
timeout 2400 python tools/ablation.py --configs c1,c2,c2d,c3,c4,c5ws,c5k --sweep-configs c2,c3,c4,c5ws,c5k --out $M/ablation.json > $M/ablation.log 2>&1
echo "ablation rc=$?"
[ -n "$GPUTESTS" ] && { timeout 2700 python -m pytest tests -m gpu -q > $M/gputests.log 2>&1; echo "gpu tests rc=$?"; tail -2 $M/gputests.log; }
du -sh gpurun_out