#!/bin/bash
# Whole GPU suite at HEAD + smoke (the driver's round-end checks).
mkdir -p gpurun_out/gputests3
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/gputests3/tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gputests3/tests.log
tail -22 gpurun_out/gputests3/tests.log
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/gputests3/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/gputests3/smoke.log
