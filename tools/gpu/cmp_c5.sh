make -j16 all > gpurun_out/make.log 2>&1
for cfg in c5ws c5k; do for eng in 1 2; do
 echo "== $cfg engine=$eng" >> gpurun_out/engines.log
 timeout 300 python tools/profile_step.py --config $cfg --sources 2048 --repeat 2 --opt engine=$eng --opt ep_min_frontier=2147483647 >> gpurun_out/engines.log 2>&1
done; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:bc_kernel -c 1 -o gpurun_out/c5ws_main python tools/profile_step.py --config c5ws --sources 512 --opt engine=1 --opt ep_min_frontier=2147483647 > gpurun_out/ncu_c5ws.log 2>&1
