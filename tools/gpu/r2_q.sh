# round 2, session Q: baseline benches on this box + ncu full captures of k_recount and k_refine at C4
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/q_env.txt
timeout 400 python bench.py --steps 30 --no-cpu-baseline --no-repartition > gpurun_out/q_bench_c2.json 2> gpurun_out/q_bench_c2.err
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/q_bench_c4.json 2> gpurun_out/q_bench_c4.err
timeout 300 python tools/recount_ab.py C4 > gpurun_out/q_rc_c4.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_recount$" -c 1 -o gpurun_out/q_recount_c4 python tools/profile_run.py C4 1 --recount > gpurun_out/q_ncu_rc.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_refine" -s 5 -c 1 -o gpurun_out/q_refine_c4 python tools/profile_step.py C4 5 > gpurun_out/q_ncu_rf.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_step" -s 5 -c 1 -o gpurun_out/q_step_c2 python tools/profile_step.py C2 6 > gpurun_out/q_ncu_st.log 2>&1
ls -la gpurun_out/
