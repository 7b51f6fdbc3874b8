#!/bin/bash
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 600 python bench.py > gpurun_out/bench_c4_check3.json 2> gpurun_out/bench_c4_check3.err
head -c 300 gpurun_out/bench_c4_check3.json; echo
timeout 1200 python bench.py --config c5k --sources 8192 --steps 3 --no-cpu-baseline > gpurun_out/bench_c5k_check3.json 2> gpurun_out/bench_c5k_check3.err
head -c 300 gpurun_out/bench_c5k_check3.json; echo
timeout 2400 python -m pytest tests -m gpu -x -q --durations=10 > gpurun_out/gputests_check3.log 2>&1; echo "tests rc=$?" >> gpurun_out/gputests_check3.log
tail -15 gpurun_out/gputests_check3.log
bash tools/gpu/sanitize.sh > gpurun_out/sanitize_summary.txt 2>&1
cat gpurun_out/sanitize_summary.txt
NOEP="--opt ep_min_frontier=2147483647"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_kernel --launch-skip 1 -c 1 -o gpurun_out/full_c4_r02b python tools/profile_step.py --config c4 --sources 4096 $NOEP > gpurun_out/ncu_c4_r02b.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:group_kernel -c 1 -o gpurun_out/full_c5k_r02b python tools/profile_step.py --config c5k --sources 512 $NOEP > gpurun_out/ncu_c5k_r02b.log 2>&1
ls -la gpurun_out/*.ncu-rep
