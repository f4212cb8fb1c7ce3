# round 2, session G: A/B of block sizes, sanitizers, launch list
set -x
for v in default t768 t1024; do
  if [ $v = default ]; then L=""; else L="IGK_LIB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 30 --no-cpu-baseline --no-repartition > gpurun_out/g_ab_c2_$v.json 2> gpurun_out/g_ab_c2_$v.err
  env $L timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/g_ab_c4_$v.json 2> gpurun_out/g_ab_c4_$v.err
done
for t in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $t python tools/sanitize_c1.py > gpurun_out/g_san_$t.txt 2>&1
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/g_launches_c2.csv python bench.py --steps 3 --warmup 3 --profile > /dev/null 2>&1
for f in gpurun_out/g_ab_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'])"; done
tail -2 gpurun_out/g_san_*.txt
