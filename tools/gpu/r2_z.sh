# round 2, session Z: item dealing A/B (packed short lists: warp-aggregated appends) + aggregated N reservations
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
IGK_LIB=$AB/libigk_deal1.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_paths.py -q -x -p no:cacheprovider -k "not 1000 and not c4 and not c5" > gpurun_out/z_pytest_deal1.txt 2>&1
tail -2 gpurun_out/z_pytest_deal1.txt
for rep in 1 2; do
for v in main deal1; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/z_bench_c2_${v}_$rep.json 2> gpurun_out/z_bench_c2_${v}_$rep.err
done
done
for v in main deal1; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/z_bench_c4_$v.json 2> gpurun_out/z_bench_c4_$v.err
done
IGK_LIB=$AB/libigk_deal1.so IGK_FLUSH=1 IGK_DEBUG_ARRIVALS=1 timeout 300 python tools/phase_profile.py 12 C2 > gpurun_out/z_phase_c2_deal1.txt 2>&1
for f in gpurun_out/z_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'])"; done
