# round 2, session AE: code-size A/B for the latency-bound C2 step (thread bucket 16 -> 8 / 4 entries) vs base (60b1d15)
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main base td8 td4; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/ae_bench_c2_${v}_$rep.json 2> gpurun_out/ae_bench_c2_${v}_$rep.err
done
done
for v in main td8; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/ae_bench_c4_$v.json 2> gpurun_out/ae_bench_c4_$v.err
done
IGK_LIB=$AB/libigk_td8.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_paths.py -q -x -p no:cacheprovider -k "not 1000 and not c4 and not c5" > gpurun_out/ae_pytest_td8.txt 2>&1
tail -2 gpurun_out/ae_pytest_td8.txt
for f in gpurun_out/ae_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'])"; done
