#!/bin/bash
mkdir -p gpurun_out
IGK_FGP_TRACE=1 PYTHONPATH=. timeout 900 python tools/fgp_time.py c1 c2 c4 > gpurun_out/n_fgp_trace.txt 2>&1
echo "rc=$?" >> gpurun_out/n_fgp_trace.txt
grep -v pass gpurun_out/n_fgp_trace.txt | tail -n 40
