#!/bin/bash
# Fast-path A/B (c1..c4 against build/base = commit 1575dc9), then the per-source parity tests.
mkdir -p gpurun_out
SPECS="c4:16384 c3:8192 c2d:0 c2:0 c1:0 c4:4096:strategy=hybrid c3:4096:strategy=hybrid c2:0:strategy=sampling,ep_min_frontier=512 c3:8192:strategy=sampling,ep_min_frontier=512" bash tools/gpu/ab.sh > gpurun_out/ab_fast1.txt 2>&1
cat gpurun_out/ab_fast1.txt
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_abi_c.py -x -q > gpurun_out/parity_fast1.log 2>&1; echo "parity rc=$?" >> gpurun_out/parity_fast1.log
tail -15 gpurun_out/parity_fast1.log
