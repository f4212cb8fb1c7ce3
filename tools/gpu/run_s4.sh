set -x
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -5 > gpurun_out/s4_pytest.txt
timeout 400 python bench.py --config C4 --steps 15 --cpu-iters 2 --no-repartition > gpurun_out/s4_bench_c4.json 2> gpurun_out/s4_bench_c4.err
timeout 300 python bench.py --steps 30 --cpu-iters 20 --no-repartition > gpurun_out/s4_bench_c2.json 2> gpurun_out/s4_bench_c2.err
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/s4_phase_c4.txt 2>&1
timeout 300 python tools/phase_profile.py 10 C3 64 0.1 > gpurun_out/s4_phase_c3.txt 2>&1
timeout 300 python tools/phase_profile.py 10 C5 > gpurun_out/s4_phase_c5.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_recount -c 1 -o gpurun_out/s4_recount_c4 python tools/profile_step.py C4 2 > gpurun_out/s4_ncu_rc.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_step -s 3 -c 1 -o gpurun_out/s4_step_c4 python tools/profile_step.py C4 5 > gpurun_out/s4_ncu_step.log 2>&1
cat gpurun_out/s4_pytest.txt
