#!/bin/bash
# Per-source engine row-split knobs on c4 (2048 sources, B200 guard): kernel ms
for s in ${SEQ:-64 128 256 1024}; do
  for w in ${WARP:-16384 65536}; do
    printf "seq_max_deg=%-4s warp_max_deg=%-6s " $s $w
    python tools/profile_step.py --config ${CFG:-c4} --sources ${N:-2048} --opt engine=1 --opt ep_min_frontier=2147483647 \
      --opt seq_max_deg=$s --opt warp_max_deg=$w 2>&1 | tail -1 | grep -o "'kernel_ms': [0-9.]*"
  done
done
