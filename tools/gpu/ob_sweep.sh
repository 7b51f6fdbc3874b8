#!/bin/bash
# Ownership-block sweep of the group engine on c5ws (BC_OWN_BLOCK, bitmap words per block).
mkdir -p gpurun_out
for ob in 8 32 128; do
  echo "== c5ws own_block=$ob" >> gpurun_out/ob.log
  BC_OWN_BLOCK=$ob timeout 300 python tools/profile_step.py --config c5ws --sources 2048 --repeat 2 --opt ep_min_frontier=2147483647 2>&1 | tail -n 1 >> gpurun_out/ob.log
done
echo "== c5k own_block=4" >> gpurun_out/ob.log
BC_OWN_BLOCK=4 timeout 300 python tools/profile_step.py --config c5k --sources 2048 --repeat 2 --opt ep_min_frontier=2147483647 2>&1 | tail -n 1 >> gpurun_out/ob.log
