#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fgp.py -x -q > gpurun_out/o_pytest_fgp.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/o_pytest_fgp.txt
PYTHONPATH=. timeout 900 python tools/fgp_time.py c1 c2 c4 > gpurun_out/o_fgp_time.txt 2>&1
echo "rc=$?" >> gpurun_out/o_fgp_time.txt
IGK_FGP_TRACE=1 PYTHONPATH=. timeout 900 python tools/fgp_time.py c2 > gpurun_out/o_fgp_trace.txt 2>&1
tail -n 5 gpurun_out/o_pytest_fgp.txt gpurun_out/o_fgp_time.txt
