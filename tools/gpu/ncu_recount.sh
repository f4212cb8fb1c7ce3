mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_recount -c 1 -o gpurun_out/s15_recount_c4 -f python tools/profile_run.py C4 3 --recount > gpurun_out/s15_ncu.log 2>&1
ncu -i gpurun_out/s15_recount_c4.ncu-rep --page source --csv > gpurun_out/s15_recount_src.csv 2>&1
ncu -i gpurun_out/s15_recount_c4.ncu-rep --page raw --csv > gpurun_out/s15_recount_raw.csv 2>&1
tail -3 gpurun_out/s15_ncu.log
