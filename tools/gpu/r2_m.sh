#!/bin/bash
# session M: NEXT-2 parity + timing
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fgp.py -x -q > gpurun_out/m_pytest_fgp.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/m_pytest_fgp.txt
echo "pytest rc=$?" >> gpurun_out/m_pytest_fgp.txt
PYTHONPATH=. timeout 900 python tools/fgp_time.py c1 c2 c4 > gpurun_out/m_fgp_time.txt 2>&1
echo "time rc=$?" >> gpurun_out/m_fgp_time.txt
tail -n 5 gpurun_out/m_pytest_fgp.txt gpurun_out/m_fgp_time.txt
