#!/bin/bash
mkdir -p gpurun_out
LIBS="new:default ggen:build/ggen/libbc.so" SPECS="c5ws:2048 c5k:2048 c4:4096" bash tools/gpu/ab_multi.sh > gpurun_out/abm_group1.txt 2>&1
cat gpurun_out/abm_group1.txt
rm -rf gpurun_out/abm
timeout 1200 python -m pytest tests/test_gpu_group.py "tests/test_gpu_scale.py::test_c5_first_1024_sources_main_phase" "tests/test_gpu_scale.py::test_dist_sum_counter_pinned_to_oracle" "tests/test_gpu_scale.py::test_c5_8192_source_invariant" -x -q > gpurun_out/group1_tests.log 2>&1; echo "rc=$?" >> gpurun_out/group1_tests.log
tail -5 gpurun_out/group1_tests.log
