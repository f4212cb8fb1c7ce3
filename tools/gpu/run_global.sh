set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_global.py -x -q 2>&1 | tail -15 > gpurun_out/s2_global.txt
timeout 300 python tools/phase_profile.py 8 C4 > gpurun_out/s2_phase_c4b.txt 2>&1
cat gpurun_out/s2_global.txt
