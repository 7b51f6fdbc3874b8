#!/bin/bash
# N1 ablation at HEAD (BC_HEAD names the commit).
mkdir -p gpurun_out/abl
make -j16 all > gpurun_out/make.log 2>&1 || { tail -20 gpurun_out/make.log; exit 1; }
timeout 2400 python tools/ablation.py --configs c1,c2,c2d,c3,c4,c5ws,c5k --sweep-configs c2,c3,c4,c5ws,c5k --out gpurun_out/abl/ablation.json > gpurun_out/abl/ablation.log 2>&1
echo "ablation rc=$?"
