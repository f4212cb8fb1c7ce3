set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/f_env.txt; nproc >> gpurun_out/f_env.txt; lscpu | grep "Model name" >> gpurun_out/f_env.txt
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 > gpurun_out/f_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.txt 2>&1
timeout 400 python bench.py > gpurun_out/f_bench_c2.json 2> gpurun_out/f_bench_c2.err
timeout 500 python bench.py --config C4 --steps 15 --cpu-iters 3 > gpurun_out/f_bench_c4.json 2> gpurun_out/f_bench_c4.err
timeout 400 python bench.py --config C5 --steps 15 --cpu-iters 3 --no-repartition > gpurun_out/f_bench_c5.json 2> /dev/null
timeout 300 python bench.py --config C3 --k 64 --frac 0.1 --steps 20 --cpu-iters 10 --no-repartition > gpurun_out/f_bench_c3.json 2> /dev/null
timeout 300 python bench.py --config C1 --steps 15 --warmup 3 --no-repartition > gpurun_out/f_bench_c1.json 2> /dev/null
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/f_bench_ref.json 2> /dev/null
timeout 300 python tools/phase_profile.py 30 C2 > gpurun_out/f_phase_c2.txt 2>&1
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/f_phase_c4.txt 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/f_launches_c2.csv python bench.py --steps 3 --warmup 3 --profile > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_step -s 3 -c 1 -o gpurun_out/f_step_c2 python tools/profile_step.py C2 5 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_apply|k_refine" -s 5 -c 2 -o gpurun_out/f_split_c4 python tools/profile_step.py C4 5 > /dev/null 2>&1
cat gpurun_out/f_pytest.txt gpurun_out/f_smoke.txt
