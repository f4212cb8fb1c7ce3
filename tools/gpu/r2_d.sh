# round 2, session D: TMA recount correctness + A/B + ncu
set -x
timeout 900 python -m pytest tests/test_gpu_store.py tests/test_gpu_paths.py -q -x -p no:cacheprovider > gpurun_out/d_pytest.txt 2>&1
timeout 300 python tools/recount_ab.py C2 > gpurun_out/d_rc_c2.txt 2>&1
timeout 600 python tools/recount_ab.py C4 > gpurun_out/d_rc_c4.txt 2>&1
timeout 600 python tools/recount_ab.py C5 > gpurun_out/d_rc_c5.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_recount" -c 2 -o gpurun_out/d_recount_c4 python tools/profile_step.py C4 1 > gpurun_out/d_ncu.log 2>&1
cat gpurun_out/d_rc_c*.txt; tail -3 gpurun_out/d_pytest.txt
