#!/bin/bash
# Engine comparison: kernel ms of one bc_compute per config and engine,
# Alg. 5 with the B200 guard (no EP level), first N sources of the config's source list.
N=${N:-4096}
for cfg in c4 c5k c5ws c3; do
 for eng in 1 2; do
  echo "== $cfg engine=$eng sources=$N"
  timeout 600 python tools/profile_step.py --config $cfg --sources $N --opt engine=$eng --opt ep_min_frontier=2147483647 2>&1 | tail -1
 done
done
