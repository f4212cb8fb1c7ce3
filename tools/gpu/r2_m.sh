#!/bin/bash
# session M: NEXT-2 parity + timing
mkdir -p gpurun_out
true
echo "pytest rc=$?" >> gpurun_out/m_pytest_fgp.txt
PYTHONPATH=. timeout 900 python tools/fgp_time.py c1 c2 c4 > gpurun_out/m_fgp_time.txt 2>&1
echo "time rc=$?" >> gpurun_out/m_fgp_time.txt
tail -n 5 gpurun_out/m_pytest_fgp.txt gpurun_out/m_fgp_time.txt
