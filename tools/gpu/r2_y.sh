# round 2, session Y: C2 per-warp F1 diagnostics (flushed L2) + ncu of the final k_recount3 at C4
set -x
mkdir -p gpurun_out
IGK_FLUSH=1 IGK_DEBUG_ARRIVALS=1 timeout 300 python tools/phase_profile.py 12 C2 > gpurun_out/y_phase_c2.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_recount3" -c 1 -o gpurun_out/y_recount3_c4 python tools/profile_run.py C4 1 --recount > gpurun_out/y_ncu_rc.log 2>&1
grep -E "F1 commit|slowest CTA" gpurun_out/y_phase_c2.txt
