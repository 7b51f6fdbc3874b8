#!/bin/bash
# Round-2 first check: build, GPU tests (incl. the parity-at-scale tests), sanitizers, bench c4.
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -x -q --durations=30 > gpurun_out/gputests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gputests.log
tail -40 gpurun_out/gputests.log
bash tools/gpu/sanitize.sh > gpurun_out/sanitize_summary.txt 2>&1
cat gpurun_out/sanitize_summary.txt
timeout 900 python bench.py > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
tail -c 3000 gpurun_out/bench_c4.json
