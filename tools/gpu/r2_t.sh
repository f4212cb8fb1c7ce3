# round 2, session T: recount3 variant A/B (interleaved), hub threshold A/B on the step, commit change parity
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main m4 nopf m4nopf; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  for c in C4 C5 C2; do env $L timeout 300 python tools/recount_ab.py $c 9 v3 >> gpurun_out/t_rc_$v.txt 2>&1; done
done
done
for rep in 1 2; do
for v in main bd256 bd128; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/t_bench_c2_${v}_$rep.json 2> gpurun_out/t_bench_c2_${v}_$rep.err
done
done
for v in main bd256; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/t_bench_c4_$v.json 2> gpurun_out/t_bench_c4_$v.err
done
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/t_pytest.txt 2>&1
grep -h v3 gpurun_out/t_rc_*.txt | head -0
for v in main m4 nopf m4nopf; do echo "== $v"; grep -h '"ms"' gpurun_out/t_rc_$v.txt | cut -c1-60; done
for f in gpurun_out/t_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'])"; done
tail -3 gpurun_out/t_pytest.txt
