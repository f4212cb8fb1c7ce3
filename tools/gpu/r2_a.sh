# round 2, session A: full GPU suite (durations), smoke, C2 bench
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/a_env.txt; nproc >> gpurun_out/a_env.txt; lscpu | grep "Model name" >> gpurun_out/a_env.txt
timeout 1700 python -m pytest tests -m gpu -q --durations=30 -p no:cacheprovider > gpurun_out/a_pytest.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/a_smoke.txt 2>&1
timeout 400 python bench.py > gpurun_out/a_bench_c2.json 2> gpurun_out/a_bench_c2.err
tail -40 gpurun_out/a_pytest.txt; cat gpurun_out/a_smoke.txt
