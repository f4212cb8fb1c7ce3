# round 2, session U: recount3 A/B (defaults now 4 CTAs/SM, no tile prefetch) vs in-thread 4 / residual unroll 4; C2 flush vs no-flush
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main in4 u4; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  for c in C4 C5 C2; do env $L timeout 300 python tools/recount_ab.py $c 9 v3 >> gpurun_out/u_rc_$v.txt 2>&1; done
done
done
timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/u_bench_c2.json 2> gpurun_out/u_bench_c2.err
timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition --no-flush > gpurun_out/u_bench_c2_noflush.json 2> gpurun_out/u_bench_c2_noflush.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_recount3" -c 1 -o gpurun_out/u_recount3_c4 python tools/profile_run.py C4 1 --recount > gpurun_out/u_ncu_rc.log 2>&1
for v in main in4 u4; do echo "== $v"; grep -h '"ms"' gpurun_out/u_rc_$v.txt | cut -c1-60; done
for f in gpurun_out/u_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'])"; done
