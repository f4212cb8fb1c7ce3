# round 2, session R: k_recount3 A/B (v3 default V=4, V=2 build, round-1 gather, TMA), ncu of v3, full GPU suite
set -x
mkdir -p gpurun_out
for c in C2 C4 C5; do
  timeout 300 python tools/recount_ab.py $c 9 v3,gather > gpurun_out/r_rc_$c.txt 2>&1
  IGK_LIB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab/libigk_v2.so timeout 300 python tools/recount_ab.py $c 9 v3 > gpurun_out/r_rc_${c}_v2.txt 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_recount3" -c 1 -o gpurun_out/r_recount3_c4 python tools/profile_run.py C4 1 --recount > gpurun_out/r_ncu_rc.log 2>&1
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider --durations=10 > gpurun_out/r_pytest.txt 2>&1
cat gpurun_out/r_rc_*.txt; tail -15 gpurun_out/r_pytest.txt
