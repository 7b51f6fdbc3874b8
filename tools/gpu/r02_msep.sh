#!/bin/bash
# Multi-source EP in the batched engine: parity, then batched WE vs batched EP vs the
# per-source / group engines (kernel ms).
mkdir -p gpurun_out
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_batched.py tests/test_gpu_parity.py -x -q -k "multi_source_ep or batched or handover" > gpurun_out/msep_tests.log 2>&1; echo "rc=$?" >> gpurun_out/msep_tests.log
tail -5 gpurun_out/msep_tests.log
LIBS="new:default" SPECS="c4:4096:engine=batched,strategy=we c4:4096:engine=batched,strategy=ep c4:4096:engine=batched,strategy=sampling,ep_min_frontier=512 c4:4096:engine=batched,strategy=sampling,ep_min_frontier=32768 c4:4096:strategy=we c5k:1024:engine=batched,strategy=we c5k:1024:engine=batched,strategy=ep c5k:1024:engine=batched,strategy=sampling,ep_min_frontier=512 c5k:1024:engine=batched,strategy=sampling,ep_min_frontier=262144 c5k:1024:strategy=we c5ws:1024:engine=batched,strategy=we c5ws:1024:engine=batched,strategy=sampling,ep_min_frontier=512 c5ws:1024:engine=batched,strategy=sampling,ep_min_frontier=1048576 c5ws:1024:strategy=we" bash tools/gpu/ab_multi.sh > gpurun_out/abm_msep.txt 2>&1
cat gpurun_out/abm_msep.txt
rm -rf gpurun_out/abm
