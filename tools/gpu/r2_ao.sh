# round 2, session AO: warp-bucket entries per lane per trip A/B (8 default, 4, 2)
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main wu4 wu2; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/ao_bench_c2_${v}_$rep.json 2> gpurun_out/ao_bench_c2_${v}_$rep.err
done
done
for v in main wu4 wu2; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/ao_bench_c4_$v.json 2> gpurun_out/ao_bench_c4_$v.err
done
for f in gpurun_out/ao_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'])"; done
