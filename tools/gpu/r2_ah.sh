# round 2, session AH: cold-code microbenchmark + ncu of the C4 split step (k_apply, k_refine) for the traffic figure
set -x
mkdir -p gpurun_out
./tools/icache_bench > gpurun_out/ah_icache.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_apply|k_refine" -s 10 -c 2 -o gpurun_out/ah_split_c4 python tools/profile_step.py C4 6 > gpurun_out/ah_ncu_c4.log 2>&1
cat gpurun_out/ah_icache.txt; tail -2 gpurun_out/ah_ncu_c4.log
