# round 2, session V: recount3 (in-thread 4 entries now default) vs V=2 tiles at 6/8 CTAs per SM; C2 step: cold paths out of line
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
for rep in 1 2; do
for v in main v2m6 v2m8; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  for c in C4 C5 C2; do env $L timeout 300 python tools/recount_ab.py $c 9 v3 >> gpurun_out/v_rc_$v.txt 2>&1; done
done
done
for rep in 1 2; do
for v in main cold; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/v_bench_c2_${v}_$rep.json 2> gpurun_out/v_bench_c2_${v}_$rep.err
done
done
timeout 900 python -m pytest tests/test_gpu_store.py tests/test_gpu_paths.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "not 1000" > gpurun_out/v_pytest.txt 2>&1
for v in main v2m6 v2m8; do echo "== $v"; grep -h '"ms"' gpurun_out/v_rc_$v.txt | cut -c1-60; done
for f in gpurun_out/v_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'])"; done
tail -2 gpurun_out/v_pytest.txt
