set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" 
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/s2_pytest.txt
timeout 300 python bench.py > gpurun_out/s2_bench_c2.json 2> gpurun_out/s2_bench_c2.err
timeout 300 python tools/phase_profile.py 30 C2 > gpurun_out/s2_phase_c2.txt 2>&1
timeout 600 python tools/phase_profile.py 8 C4 > gpurun_out/s2_phase_c4.txt 2>&1
cat gpurun_out/s2_pytest.txt; tail -c 600 gpurun_out/s2_bench_c2.json
