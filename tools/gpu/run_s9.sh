set -x
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/s9_pytest.txt
timeout 400 python bench.py > gpurun_out/s9_bench_c2.json 2> gpurun_out/s9_bench_c2.err
timeout 400 python bench.py --config C4 --steps 15 --cpu-iters 3 > gpurun_out/s9_bench_c4.json 2> gpurun_out/s9_bench_c4.err
timeout 300 python tools/phase_profile.py 30 C2 > gpurun_out/s9_phase_c2.txt 2>&1
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/s9_phase_c4.txt 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s9_launches_c2.csv python bench.py --steps 3 --warmup 3 --profile > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s9_launches_c4.csv python bench.py --config C4 --steps 3 --warmup 3 --profile > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_step -s 3 -c 1 -o gpurun_out/s9_step_c2 python tools/profile_step.py C2 5 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_apply|k_refine" -s 6 -c 2 -o gpurun_out/s9_split_c4 python tools/profile_step.py C4 5 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_recount -c 1 -o gpurun_out/s9_recount_c4 python tools/profile_step.py C4 2 > /dev/null 2>&1
cat gpurun_out/s9_pytest.txt
