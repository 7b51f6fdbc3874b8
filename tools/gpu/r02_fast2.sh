#!/bin/bash
mkdir -p gpurun_out
LIBS="base:build/base/libbc.so new:default" SPECS="c4:4096 c4:4096:succ_bits=-1 c3:4096 c3:4096:succ_bits=-1 c2d:16384 c2d:16384:succ_bits=-1 c2:16384 c1:0" bash tools/gpu/ab_multi.sh > gpurun_out/abm_fast3.txt 2>&1
cat gpurun_out/abm_fast3.txt
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_abi_c.py "tests/test_gpu_scale.py::test_c4_bench_workload_elementwise" "tests/test_gpu_scale.py::test_full_config_source_sets" -x -q > gpurun_out/parity_fast3.log 2>&1; echo "parity rc=$?" >> gpurun_out/parity_fast3.log
tail -15 gpurun_out/parity_fast3.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_c4_fast3.json 2> gpurun_out/bench_c4_fast3.err
head -c 600 gpurun_out/bench_c4_fast3.json
